# call 35: fused populate+pin by default: host-image / concurrent-register / multirank / parity GPU tests + C3 bench (setup_s)
mkdir -p gpurun_out
( time timeout 1500 python -m pytest tests/test_gpu_host_image.py tests/test_gpu_concurrent_register.py tests/test_gpu_multirank.py tests/test_gpu_parity.py -q -x ) > gpurun_out/a35_tests.txt 2>&1; echo EXIT=$? >> gpurun_out/a35_tests.txt
timeout 900 python bench.py > gpurun_out/a35_bench.json 2> gpurun_out/a35_bench.err; echo EXIT=$? >> gpurun_out/a35_bench.err
echo done
