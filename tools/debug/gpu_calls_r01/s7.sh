# session-2 call 7: ncclCommShrink with the parent retired instead of freed, during an emulated hang
mkdir -p gpurun_out
NCCL_DEBUG=WARN timeout 150 python tools/debug_nccl_shrink.py 1 > gpurun_out/s7_shrink_hang.log 2>&1
timeout 600 python -m pytest tests/test_gpu_hang_collective.py tests/test_gpu_bench_multirank.py -q > gpurun_out/s7_tests.log 2>&1; echo EXIT=$? >> gpurun_out/s7_tests.log
echo done
