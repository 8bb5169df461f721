# call 22: NEXT-4 durable tier against the disk's own O_DIRECT rate (tools/durable_bench.py raw_disk)
mkdir -p gpurun_out
timeout 900 python tools/durable_bench.py --config C2 > gpurun_out/a22_durable.json 2> gpurun_out/a22_durable.err; echo EXIT=$? >> gpurun_out/a22_durable.err
echo done
