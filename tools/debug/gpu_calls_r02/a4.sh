# call 4: K2/K1 variant round-robin sweep 2 around T512 U4 b4, 8 GiB launches
mkdir -p gpurun_out
K2V_SWEEP2=1 timeout 900 ./tools/k2_variants 8192 15 > gpurun_out/a4_k2_rr2.txt 2>&1
echo done
