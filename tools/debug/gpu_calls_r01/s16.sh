# session-3 call 16: kernel-parameter-size probe for the per-launch penalty under a concurrent D2H;
# kbench K2 reference at 256 MiB; bench with the all-cores cpu_baseline
mkdir -p gpurun_out
timeout 300 tools/param_probe 256 > gpurun_out/s16_param_probe.txt 2>&1; echo EXIT=$? >> gpurun_out/s16_param_probe.txt
timeout 300 tools/kbench 256 8192 2 > gpurun_out/s16_kbench.txt 2>&1; echo EXIT=$? >> gpurun_out/s16_kbench.txt
timeout 600 python bench.py --steps 3 --warmup 3 > gpurun_out/s16_bench.json 2> gpurun_out/s16_bench.err
nproc > gpurun_out/s16_nproc.txt; lscpu | head -20 >> gpurun_out/s16_nproc.txt
echo done
