# call 5: library kernels with per-mode CTA shapes: harness, parity tests, C3 bench
mkdir -p gpurun_out
timeout 600 ./tools/k2_variants 8192 15 > gpurun_out/a5_k2_rr.txt 2>&1
( time timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_scenarios.py -x -q ) > gpurun_out/a5_gpu_tests.txt 2>&1; echo EXIT=$? >> gpurun_out/a5_gpu_tests.txt
timeout 900 python bench.py > gpurun_out/a5_bench.json 2> gpurun_out/a5_bench.err; echo EXIT=$? >> gpurun_out/a5_bench.err
echo done
