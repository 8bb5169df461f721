# session-2 call 5: kernel span instrumentation + 4 GiB bench slots: full GPU suite, default bench
set -x
mkdir -p gpurun_out
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/s5_gpu_tests.log 2>&1; echo EXIT=$? >> gpurun_out/s5_gpu_tests.log
timeout 400 python bench.py > gpurun_out/s5_bench.json 2> gpurun_out/s5_bench.err
echo done
