# call 26: bounce-buffer stage-in with 8 / 16 / 24 I/O threads
mkdir -p gpurun_out
for t in 8 16 24; do
  JITC_DURABLE_THREADS=$t timeout 900 python tools/durable_bench.py --config C2 >> gpurun_out/a26_durable.json 2>> gpurun_out/a26_durable.err; echo EXIT=$? >> gpurun_out/a26_durable.err
done
echo done
