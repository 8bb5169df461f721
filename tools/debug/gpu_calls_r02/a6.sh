# call 6: segment size 32/64/128 KiB x batch, library vs harness (round robin)
mkdir -p gpurun_out
for kib in 32 64 128; do
  echo "### segment $kib KiB" >> gpurun_out/a6_seg_sweep.txt
  K2V_SWEEP3=1 K2V_SEG_KIB=$kib timeout 300 ./tools/k2_variants 8192 11 >> gpurun_out/a6_seg_sweep.txt 2>&1
done
echo done
