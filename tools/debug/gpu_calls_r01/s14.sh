# session-3 call 14b: TMA-staged K2 variants (tools/tma_bench.cu) vs the library's LDG.128 K2, alone and
# next to a concurrent D2H; ncu of the best per-warp variant
mkdir -p gpurun_out
timeout 300 tools/tma_bench 4096 16384 > gpurun_out/s14_tma_4g.txt 2>&1; echo EXIT=$? >> gpurun_out/s14_tma_4g.txt
timeout 300 tools/tma_bench 256 8192 > gpurun_out/s14_tma_256m.txt 2>&1; echo EXIT=$? >> gpurun_out/s14_tma_256m.txt
echo done
