# session-3 call 13: full GPU suite + smoke + default bench in the restored tree; sanitizers and C3 / N=2 benches
# lost with the previous session's s12 call
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv > gpurun_out/s13_smi.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s13_smoke.log 2>&1; echo EXIT=$? >> gpurun_out/s13_smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/s13_gpu_tests.log 2>&1; echo EXIT=$? >> gpurun_out/s13_gpu_tests.log
timeout 400 python bench.py > gpurun_out/s13_bench.json 2> gpurun_out/s13_bench.err
timeout 300 python bench.py --impl reference --steps 2 --warmup 3 > gpurun_out/s13_bench_ref.json 2> gpurun_out/s13_bench_ref.err
timeout 900 python bench.py --config C3 --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/s13_bench_c3.json 2> gpurun_out/s13_bench_c3.err
JITC_BENCH_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29513 \
  bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu-baseline --hang-ctas 0 > gpurun_out/s13_bench_c2_n2share.json 2> gpurun_out/s13_bench_c2_n2share.err
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 900 $CS --tool racecheck python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s13_racecheck.log 2>&1; echo EXIT=$? >> gpurun_out/s13_racecheck.log
timeout 900 $CS --tool synccheck python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s13_synccheck.log 2>&1; echo EXIT=$? >> gpurun_out/s13_synccheck.log
echo done
