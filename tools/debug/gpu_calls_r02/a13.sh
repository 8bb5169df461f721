# call 13: does SM zero-copy traffic add host-link bandwidth on top of the copy engine? (tools/link_mix_probe.cu)
mkdir -p gpurun_out
timeout 300 ./tools/link_mix_probe 8 592 > gpurun_out/a13_link_mix.txt 2>&1
timeout 300 ./tools/link_mix_probe 8 148 >> gpurun_out/a13_link_mix.txt 2>&1
timeout 300 ./tools/link_mix_probe 8 1184 >> gpurun_out/a13_link_mix.txt 2>&1
echo done
