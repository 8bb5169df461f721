# round 2 session 3, call 1: regression of the restored tree (tests, smoke, default bench)
mkdir -p gpurun_out
nvidia-smi -L > gpurun_out/a1_smi.txt 2>&1
( time timeout 1500 python -m pytest tests -m gpu -x -q ) > gpurun_out/a1_gpu_tests.txt 2>&1; echo EXIT=$? >> gpurun_out/a1_gpu_tests.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/a1_smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/a1_bench.json 2> gpurun_out/a1_bench.err; echo EXIT=$? >> gpurun_out/a1_bench.err
echo done
