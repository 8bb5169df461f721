# call 43: grid sizes computed at jitc_create (preload): watchdog / hang / parity tests + smoke
mkdir -p gpurun_out
timeout 1500 python -m pytest tests/test_gpu_watchdog.py tests/test_gpu_hang_collective.py tests/test_gpu_parity.py -q > gpurun_out/a43_tests.txt 2>&1; echo EXIT=$? >> gpurun_out/a43_tests.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/a43_smoke.txt 2>&1; echo EXIT=$? >> gpurun_out/a43_smoke.txt
echo done
