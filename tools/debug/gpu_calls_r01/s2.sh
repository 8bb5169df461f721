set -x
python tools/nccl_same_gpu.py > gpurun_out/s2_nccl_probe.log 2>&1; echo probe=$? >> gpurun_out/s2_nccl_probe.log
for p in 0 256 64 1024 0 256; do
  JITC_COPY_PIECE_MB=$p timeout 300 python bench.py --steps 4 --warmup 3 --no-cpu-baseline --hang-ctas 0 > gpurun_out/s2_bench_piece$p.json 2>gpurun_out/s2_bench_piece$p.err
done
timeout 900 python -m pytest tests/test_gpu_multirank.py tests/test_gpu_bench_multirank.py -x -q -k nccl > gpurun_out/s2_nccl_tests.log 2>&1; echo EXIT=$? >> gpurun_out/s2_nccl_tests.log
