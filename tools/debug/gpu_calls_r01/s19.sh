# session-3 call 19: round-end regression of the final tree: full GPU suite, smoke, default bench (N=1, C2),
# reference arm, ncu launch list of the same bench command
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s19_smoke.log 2>&1; echo EXIT=$? >> gpurun_out/s19_smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/s19_gpu_tests.log 2>&1; echo EXIT=$? >> gpurun_out/s19_gpu_tests.log
timeout 600 python bench.py > gpurun_out/s19_bench.json 2> gpurun_out/s19_bench.err
timeout 300 python bench.py --impl reference > gpurun_out/s19_bench_ref.json 2> gpurun_out/s19_bench_ref.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:seg_kernel -c 400 --csv \
  --log-file gpurun_out/s19_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --hang-ctas 0 > gpurun_out/s19_ncu_bench.log 2>&1
echo done
