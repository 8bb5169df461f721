# call 24: O_DIRECT read destination probe (tools/disk_dest_probe.py)
mkdir -p gpurun_out
timeout 900 python tools/disk_dest_probe.py /tmp/ddp 16 8 > gpurun_out/a24_disk_dest.txt 2>&1; echo EXIT=$? >> gpurun_out/a24_disk_dest.txt
rm -rf /tmp/ddp
echo done
