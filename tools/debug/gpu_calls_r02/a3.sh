# call 3: K2 variant round-robin sweep (drift-robust), 8 GiB launches, 15 passes
mkdir -p gpurun_out
timeout 900 ./tools/k2_variants 8192 15 > gpurun_out/a3_k2_rr.txt 2>&1
echo done
