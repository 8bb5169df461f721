# call 41: capture pipeline across groups (EUNSTABLE in the second group, no partial commit) + commit semantics tests
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_commit_semantics.py tests/test_gpu_transient.py tests/test_gpu_watchdog.py -q > gpurun_out/a41_tests.txt 2>&1; echo EXIT=$? >> gpurun_out/a41_tests.txt
echo done
