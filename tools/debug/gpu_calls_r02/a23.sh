# call 23: durable tier I/O threads 8 / 16 / 32 (JITC_DURABLE_THREADS) vs the raw O_DIRECT rate
mkdir -p gpurun_out
for t in 8 16 32; do
  JITC_DURABLE_THREADS=$t timeout 900 python tools/durable_bench.py --config C2 >> gpurun_out/a23_durable.json 2>> gpurun_out/a23_durable.err; echo EXIT=$? >> gpurun_out/a23_durable.err
done
echo done
