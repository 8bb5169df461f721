# session-2 call 11: new tests (attach errors, full-size parity at 4 GiB rounds, N=1 bench contract), bench with the
# watchdog variant, ncu launch list of the current bench command and a full-set capture at 4 GiB launches
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_gpu_fanout.py tests/test_gpu_parity.py tests/test_gpu_bench_multirank.py -q -k "attach or full_size or contract" > gpurun_out/s11_tests.log 2>&1; echo EXIT=$? >> gpurun_out/s11_tests.log
timeout 400 python bench.py > gpurun_out/s11_bench.json 2> gpurun_out/s11_bench.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:seg_kernel -c 400 --csv \
  --log-file gpurun_out/s11_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --hang-ctas 0 > gpurun_out/s11_ncu_bench.log 2>&1
PROF_SLOT_MB=4096 PROF_STAGING_MB=8192 PROF_BYTES=$((8<<30)) timeout 900 ncu --set full --clock-control none --import-source on -k regex:seg_kernel -s 1 -c 4 \
  -o gpurun_out/s11_prof python tools/prof_kernels.py > gpurun_out/s11_prof.log 2>&1
echo done
