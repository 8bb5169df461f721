# call 8: library kernel via libjitc.so vs the same source compiled into the harness TU
mkdir -p gpurun_out
echo "### libjitc.so" > gpurun_out/a8_lib_vs_inc.txt
K2V_SWEEP3=1 K2V_SEG_KIB=128 timeout 300 ./tools/k2_variants 8192 11 >> gpurun_out/a8_lib_vs_inc.txt 2>&1
echo "### included" >> gpurun_out/a8_lib_vs_inc.txt
K2V_SWEEP3=1 K2V_SEG_KIB=128 timeout 300 ./tools/k2_variants_inc 8192 11 >> gpurun_out/a8_lib_vs_inc.txt 2>&1
echo done
