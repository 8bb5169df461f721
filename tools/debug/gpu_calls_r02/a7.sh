# call 7: 128 KiB segments + per-mode shapes: harness, full GPU suite, smoke, C3 bench
mkdir -p gpurun_out
K2V_SWEEP3=1 K2V_SEG_KIB=128 timeout 300 ./tools/k2_variants 8192 11 > gpurun_out/a7_k2_rr.txt 2>&1
( time timeout 1500 python -m pytest tests -m gpu -x -q ) > gpurun_out/a7_gpu_tests.txt 2>&1; echo EXIT=$? >> gpurun_out/a7_gpu_tests.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/a7_smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/a7_bench.json 2> gpurun_out/a7_bench.err; echo EXIT=$? >> gpurun_out/a7_bench.err
echo done
