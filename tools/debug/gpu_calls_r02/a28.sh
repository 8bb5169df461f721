# call 28: stage-in A/B on one box: no bounce / one / two bounce buffers per thread, 3 rounds each, interleaved
mkdir -p gpurun_out
for rep in 1 2 3; do
  for b in 0 1 2; do
    echo "bounce=$b" >> gpurun_out/a28_durable.json
    JITC_DURABLE_BOUNCE=$b timeout 900 python tools/durable_bench.py --config C2 >> gpurun_out/a28_durable.json 2>> gpurun_out/a28_durable.err
  done
done
echo done
