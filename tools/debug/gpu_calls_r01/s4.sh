# session-2 call 4: default bench, slot-size experiment for K2's live roofline, ncu launch list of the bench command, C3
set -x
mkdir -p gpurun_out
timeout 400 python bench.py > gpurun_out/s4_bench_default.json 2> gpurun_out/s4_bench_default.err
timeout 300 python bench.py --steps 4 --warmup 3 --no-cpu-baseline --hang-ctas 0 --slot 4096 > gpurun_out/s4_bench_slot4096.json 2> gpurun_out/s4_bench_slot4096.err
timeout 300 python bench.py --steps 4 --warmup 3 --no-cpu-baseline --hang-ctas 0 --slot 4096 --staging 16384 > gpurun_out/s4_bench_slot4096_stg16.json 2> gpurun_out/s4_bench_slot4096_stg16.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:seg_kernel -c 400 --csv \
  --log-file gpurun_out/s4_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --hang-ctas 0 > gpurun_out/s4_ncu_bench.log 2>&1
timeout 900 python bench.py --config C3 --steps 2 --warmup 3 --no-cpu-baseline --hang-ctas 0 > gpurun_out/s4_bench_c3.json 2> gpurun_out/s4_bench_c3.err
echo done
