# session-3 call 38: C3 (Llama-3-8B, 128.5 GB) N=1 with the final tree; C2 N=2 sharing one GPU (functional, PEER variant)
mkdir -p gpurun_out
timeout 1200 python bench.py --config C3 --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/s38_bench_c3.json 2> gpurun_out/s38_bench_c3.err
JITC_BENCH_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29551 \
  bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu-baseline --hang-ctas 0 > gpurun_out/s38_bench_c2_n2share.json 2> gpurun_out/s38_bench_c2_n2share.err
echo done
