# call 2: K2 streaming-core variant sweep (tools/k2_variants.cu), 8 GiB launches
mkdir -p gpurun_out
timeout 600 ./tools/k2_variants 8192 10 > gpurun_out/a2_k2_variants.txt 2>&1
timeout 300 ./tools/k2_variants 1024 20 > gpurun_out/a2_k2_variants_1g.txt 2>&1
echo done
