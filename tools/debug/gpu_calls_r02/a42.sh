# call 42: commit agrees on "every writer captured at v*" before anyone writes: commit / multi-rank / dead-peer GPU tests
mkdir -p gpurun_out
( time timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_commit_semantics.py tests/test_gpu_multirank.py tests/test_gpu_writer_death.py tests/test_gpu_hang_collective.py tests/test_gpu_scenarios.py tests/test_gpu_fanout.py tests/test_gpu_bench_multirank.py -q ) > gpurun_out/a42_tests.txt 2>&1; echo EXIT=$? >> gpurun_out/a42_tests.txt
echo done
