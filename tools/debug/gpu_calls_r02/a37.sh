# call 37: does a C3 bench right after the parity suite (with its 128 GB every-chunk images) run slow?
# same sequence as call 35, then benches with fused (default) and two-phase pinning
mkdir -p gpurun_out
free -g > gpurun_out/a37_mem.txt
( time timeout 1500 python -m pytest tests/test_gpu_host_image.py tests/test_gpu_concurrent_register.py tests/test_gpu_multirank.py tests/test_gpu_parity.py -q -x ) > gpurun_out/a37_tests.txt 2>&1; echo EXIT=$? >> gpurun_out/a37_tests.txt
free -g >> gpurun_out/a37_mem.txt; cat /proc/meminfo | head -25 >> gpurun_out/a37_mem.txt
for f in 1 0; do
  echo "fused=$f" >> gpurun_out/a37_ab.txt
  JITC_PIN_FUSED=$f timeout 900 python bench.py --no-cpu-baseline > gpurun_out/a37_tmp.json 2>> gpurun_out/a37_ab.err
  tail -1 gpurun_out/a37_tmp.json >> gpurun_out/a37_ab.txt
  free -g >> gpurun_out/a37_mem.txt
done
echo done
