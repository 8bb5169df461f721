# session-3 call 14: TMA-staged K2 experiment (tools/tma_bench.cu) vs the library's LDG.128 K2, alone and
# next to a concurrent D2H; ncu full-set capture of one launch of each
mkdir -p gpurun_out
timeout 300 tools/tma_bench 4096 16384 > gpurun_out/s14_tma_4g.txt 2>&1; echo EXIT=$? >> gpurun_out/s14_tma_4g.txt
timeout 300 tools/tma_bench 256 8192 > gpurun_out/s14_tma_256m.txt 2>&1; echo EXIT=$? >> gpurun_out/s14_tma_256m.txt
timeout 600 ncu --set full --clock-control none -k regex:"tma_pack|seg_kernel" -s 6 -c 2 -o gpurun_out/s14_tma tools/tma_bench 1024 4096 > gpurun_out/s14_ncu.log 2>&1
echo done
