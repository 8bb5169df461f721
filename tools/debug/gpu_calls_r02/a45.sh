# call 45: final regression of the round-2 tree: full GPU suite, smoke, default bench (C3, N=1), reference arm
mkdir -p gpurun_out
( time timeout 1800 python -m pytest tests -m gpu -q ) > gpurun_out/a45_gpu_tests.txt 2>&1; echo EXIT=$? >> gpurun_out/a45_gpu_tests.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/a45_smoke.txt 2>&1; echo EXIT=$? >> gpurun_out/a45_smoke.txt
( time timeout 900 python bench.py > gpurun_out/a45_bench.json ) 2> gpurun_out/a45_bench.err; echo EXIT=$? >> gpurun_out/a45_bench.err
( time timeout 600 python bench.py --impl reference > gpurun_out/a45_ref.json ) 2> gpurun_out/a45_ref.err; echo EXIT=$? >> gpurun_out/a45_ref.err
echo done
