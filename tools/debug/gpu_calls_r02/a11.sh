# call 11: compute-sanitizer over the round-2 kernel shapes (128 KiB segments, 512-thread CTAs)
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 1500 $CS --tool memcheck --leak-check no python -m pytest tests/test_gpu_parity.py -q \
  -k "k1_digests_match_oracle or capture_restore_bit_exact or edge_empty or k4_ or k1_c1_full or corrupt_host_image or hbm_bitflip" > gpurun_out/a11_memcheck_parity.log 2>&1; echo EXIT=$? >> gpurun_out/a11_memcheck_parity.log
timeout 900 $CS --tool memcheck --leak-check no --target-processes all python -m pytest tests/test_gpu_peer_pull.py -q > gpurun_out/a11_memcheck_pull.log 2>&1; echo EXIT=$? >> gpurun_out/a11_memcheck_pull.log
timeout 900 $CS --tool racecheck python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/a11_racecheck.log 2>&1; echo EXIT=$? >> gpurun_out/a11_racecheck.log
timeout 900 $CS --tool synccheck python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/a11_synccheck.log 2>&1; echo EXIT=$? >> gpurun_out/a11_synccheck.log
echo done
