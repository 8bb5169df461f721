# call 32: ncu launch list of the default bench command with the final pipelines
mkdir -p gpurun_out
timeout 1500 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:seg_kernel -c 400 --csv \
  --log-file gpurun_out/a32_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --hang-ctas 0 > gpurun_out/a32_ncu_bench.log 2>&1
echo done
