# session-2 call 9: NCCL warm-up at comm_init -> shrink + first collective during an emulated hang
mkdir -p gpurun_out
NCCL_DEBUG=WARN timeout 150 python tools/debug_nccl_shrink.py 1 0 1 > gpurun_out/s9_shrink_1_0_1.log 2>&1
timeout 900 python -m pytest tests/test_gpu_hang_collective.py tests/test_gpu_multirank.py tests/test_gpu_fanout.py -q -k "nccl" > gpurun_out/s9_tests.log 2>&1; echo EXIT=$? >> gpurun_out/s9_tests.log
echo done
