# call 9: ncu --set full of the library K2 vs the harness's best K2 (T512 U4 b1), 128 KiB segments
mkdir -p gpurun_out
K2V_SWEEP3=1 K2V_SEG_KIB=128 timeout 600 ncu --set full --clock-control none --import-source on \
  --kernel-name-base mangled -k 'regex:seg_kernelILi2E|seg_kernelILi1E|k2vILi512ELi4ELi1ELi1ELi0ELi1ELi1E|k2vILi256ELi8ELi1ELi1ELi3ELi1ELi2E' -c 4 \
  -o gpurun_out/a9_k2 -f ./tools/k2_variants_inc 8192 1 > gpurun_out/a9_ncu.log 2>&1
echo done
