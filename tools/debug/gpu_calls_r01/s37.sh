# session-3 call 37: regression after the dead-peer work: smoke, full GPU suite, default bench, reference arm
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s37_smoke.log 2>&1; echo EXIT=$? >> gpurun_out/s37_smoke.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/s37_gpu_tests.log 2>&1; echo EXIT=$? >> gpurun_out/s37_gpu_tests.log
timeout 600 python bench.py > gpurun_out/s37_bench.json 2> gpurun_out/s37_bench.err
timeout 300 python bench.py --impl reference > gpurun_out/s37_bench_ref.json 2> gpurun_out/s37_bench_ref.err
echo done
