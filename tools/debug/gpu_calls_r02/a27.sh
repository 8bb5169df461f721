# call 27: stage-in with double bounce buffers (memcpy overlapped with the next read); durable GPU tests + durable bench
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_durable.py -q > gpurun_out/a27_tests.txt 2>&1; echo EXIT=$? >> gpurun_out/a27_tests.txt
timeout 900 python tools/durable_bench.py --config C2 > gpurun_out/a27_durable.json 2> gpurun_out/a27_durable.err; echo EXIT=$? >> gpurun_out/a27_durable.err
cp tools/disk_dest_probe.py /dev/null
echo done
