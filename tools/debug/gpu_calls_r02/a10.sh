# call 10: ncu evidence for the round-2 kernel shapes:
#  (1) launch list of the default bench command (C3), (2) --set full of K1/K2/K3 at 8 GiB launches (prof_kernels.py)
mkdir -p gpurun_out
PROF_BYTES=$((8<<30)) PROF_STAGING_MB=16384 PROF_SLOT_MB=8192 PROF_REPS=1 timeout 900 \
  ncu --set full --clock-control none --import-source on -k regex:seg_kernel -c 4 \
  -o gpurun_out/a10_full -f python tools/prof_kernels.py > gpurun_out/a10_full.log 2>&1
timeout 1500 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:seg_kernel -c 400 --csv \
  --log-file gpurun_out/a10_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --hang-ctas 0 > gpurun_out/a10_ncu_bench.log 2>&1
echo done
