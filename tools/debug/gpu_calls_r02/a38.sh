# call 38: bench with the bounded settle loop (C2 N=1, and a 2-rank dry run)
mkdir -p gpurun_out
timeout 900 python bench.py --config C2 --steps 3 --no-cpu-baseline > gpurun_out/a38_c2.json 2> gpurun_out/a38_c2.err; echo EXIT=$? >> gpurun_out/a38_c2.err
JITC_BENCH_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --master-addr 127.0.0.1 --nproc-per-node 2 --master-port 29581 bench.py --gpus 2 --config C1 --steps 3 --warmup 3 \
  --no-cpu-baseline --staging 512 --slot 128 > gpurun_out/a38_c1_n2.json 2> gpurun_out/a38_c1_n2.err; echo EXIT=$? >> gpurun_out/a38_c1_n2.err
echo done
