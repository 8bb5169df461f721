# session-2 call 3: fan-out GPU tests, full GPU suite, copy-piece refinement, ncu (launch list + full set)
set -x
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_fanout.py -x -q > gpurun_out/s3_fanout.log 2>&1; echo EXIT=$? >> gpurun_out/s3_fanout.log
timeout 1800 python -m pytest tests -m gpu -q > gpurun_out/s3_gpu_tests.log 2>&1; echo EXIT=$? >> gpurun_out/s3_gpu_tests.log
for p in 32 16 64 128; do
  JITC_COPY_PIECE_MB=$p timeout 300 python bench.py --steps 4 --warmup 3 --no-cpu-baseline --hang-ctas 0 > gpurun_out/s3_bench_piece$p.json 2>gpurun_out/s3_bench_piece$p.err
done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -c 400 --csv \
  --log-file gpurun_out/s3_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --hang-ctas 0 > gpurun_out/s3_ncu_bench.log 2>&1
PROF_SLOT_MB=2048 PROF_STAGING_MB=4096 PROF_BYTES=$((4<<30)) timeout 900 ncu --set full --clock-control none --import-source on -k regex:seg_kernel -s 2 -c 6 \
  -o gpurun_out/s3_prof python tools/prof_kernels.py > gpurun_out/s3_prof.log 2>&1
echo done
