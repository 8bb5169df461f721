# session-2 call 10: full GPU suite after the NCCL changes; default bench; N=2 bench on one GPU (both transports) for the new fields
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/s10_gpu_tests.log 2>&1; echo EXIT=$? >> gpurun_out/s10_gpu_tests.log
timeout 400 python bench.py > gpurun_out/s10_bench.json 2> gpurun_out/s10_bench.err
for t in ipc nccl; do
JITC_BENCH_SHARE_GPU=1 timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29511 \
  bench.py --gpus 2 --steps 3 --warmup 3 --config C1 --no-cpu-baseline --staging 256 --slot 64 --hang-ctas 0 --transport $t > gpurun_out/s10_bench_n2_$t.json 2> gpurun_out/s10_bench_n2_$t.err
done
echo done
