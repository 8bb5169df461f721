# call 29: bench with the read-only HBM calibration (K1 reported against it too)
mkdir -p gpurun_out
timeout 900 python bench.py --config C2 --steps 3 --no-cpu-baseline > gpurun_out/a29_c2.json 2> gpurun_out/a29_c2.err; echo EXIT=$? >> gpurun_out/a29_c2.err
echo done
