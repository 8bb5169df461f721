# session-3 call 18: 8- and 4-rank dry runs of bench.py's N>1 path on one GPU (JITC_BENCH_SHARE_GPU, functional
# only): C1 with 8 ranks over IPC, C1 with 4 ranks over NCCL (socket transport), C2 with 4 ranks over IPC
mkdir -p gpurun_out
export JITC_BENCH_SHARE_GPU=1
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 8 --master-addr 127.0.0.1 --master-port 29521 \
  bench.py --gpus 8 --config C1 --steps 3 --warmup 3 --no-cpu-baseline --staging 512 --slot 128 --no-calibrate \
  > gpurun_out/s18_c1_n8_ipc.json 2> gpurun_out/s18_c1_n8_ipc.err; echo EXIT=$? >> gpurun_out/s18_c1_n8_ipc.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 4 --master-addr 127.0.0.1 --master-port 29522 \
  bench.py --gpus 4 --config C1 --steps 3 --warmup 3 --no-cpu-baseline --staging 512 --slot 128 --no-calibrate \
  --transport nccl > gpurun_out/s18_c1_n4_nccl.json 2> gpurun_out/s18_c1_n4_nccl.err; echo EXIT=$? >> gpurun_out/s18_c1_n4_nccl.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 4 --master-addr 127.0.0.1 --master-port 29523 \
  bench.py --gpus 4 --config C2 --steps 3 --warmup 3 --no-cpu-baseline --staging 4096 --slot 1024 --hang-ctas 0 \
  > gpurun_out/s18_c2_n4_ipc.json 2> gpurun_out/s18_c2_n4_ipc.err; echo EXIT=$? >> gpurun_out/s18_c2_n4_ipc.err
echo done
