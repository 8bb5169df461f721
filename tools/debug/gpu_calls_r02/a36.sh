# call 36: C3 bench A/B on one box: two-phase pinning (JITC_PIN_FUSED=0) vs fused populate+pin (=1), twice each
mkdir -p gpurun_out
for f in 0 1 0 1; do
  echo "fused=$f" >> gpurun_out/a36_ab.txt
  JITC_PIN_FUSED=$f timeout 900 python bench.py --no-cpu-baseline > gpurun_out/a36_tmp.json 2>> gpurun_out/a36_ab.err
  tail -1 gpurun_out/a36_tmp.json >> gpurun_out/a36_ab.txt
done
echo done
