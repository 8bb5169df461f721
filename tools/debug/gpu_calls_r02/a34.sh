# call 34: setup of the C3 image: populate-then-pin vs per-piece populate+pin (JITC_PIN_FUSED)
mkdir -p gpurun_out
for rep in 1 2; do
  for f in 0 1; do
    JITC_PIN_FUSED=$f timeout 600 python tools/setup_probe.py C3 >> gpurun_out/a34_setup.txt 2>&1
  done
done
echo done
