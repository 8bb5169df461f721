# session-3 call 27: bench.py's new PEER-restore variant at N > 1 (ranks share one GPU; functional):
# the 2-rank bench tests over both transports, then C1 with 4 ranks (IPC, NCCL) and C2 with 2 ranks (IPC)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_bench_multirank.py -q > gpurun_out/s27_tests.log 2>&1; echo EXIT=$? >> gpurun_out/s27_tests.log
export JITC_BENCH_SHARE_GPU=1
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 4 --master-addr 127.0.0.1 --master-port 29531 \
  bench.py --gpus 4 --config C1 --steps 3 --warmup 3 --no-cpu-baseline --staging 512 --slot 128 --no-calibrate \
  > gpurun_out/s27_c1_n4_ipc.json 2> gpurun_out/s27_c1_n4_ipc.err; echo EXIT=$? >> gpurun_out/s27_c1_n4_ipc.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 4 --master-addr 127.0.0.1 --master-port 29532 \
  bench.py --gpus 4 --config C1 --steps 3 --warmup 3 --no-cpu-baseline --staging 512 --slot 128 --no-calibrate \
  --transport nccl > gpurun_out/s27_c1_n4_nccl.json 2> gpurun_out/s27_c1_n4_nccl.err; echo EXIT=$? >> gpurun_out/s27_c1_n4_nccl.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 \
  bench.py --gpus 2 --config C2 --steps 3 --warmup 3 --no-cpu-baseline --hang-ctas 0 \
  > gpurun_out/s27_c2_n2_ipc.json 2> gpurun_out/s27_c2_n2_ipc.err; echo EXIT=$? >> gpurun_out/s27_c2_n2_ipc.err
echo done
