# call 12: transparent huge pages for the shared image? (tools/thp_probe.py)
mkdir -p gpurun_out
timeout 600 python tools/thp_probe.py 16 8 > gpurun_out/a12_thp_probe.txt 2>&1; echo EXIT=$? >> gpurun_out/a12_thp_probe.txt
echo done
