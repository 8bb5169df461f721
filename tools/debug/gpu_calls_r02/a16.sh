# call 16: bench with a private pinned image (N = 1 fallback when /dev/shm is too small)
mkdir -p gpurun_out
timeout 900 python bench.py --config C2 --private-image --steps 3 --warmup 3 > gpurun_out/a16_c2_private.json 2> gpurun_out/a16_c2_private.err; echo EXIT=$? >> gpurun_out/a16_c2_private.err
echo done
