# call 31: regression after the PEER / fan-out plan and stage-in changes: full GPU suite, smoke, default bench (C3, N=1), reference arm
mkdir -p gpurun_out
( time timeout 1800 python -m pytest tests -m gpu -q ) > gpurun_out/a31_gpu_tests.txt 2>&1; echo EXIT=$? >> gpurun_out/a31_gpu_tests.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" > gpurun_out/a31_smoke.txt 2>&1; echo EXIT=$? >> gpurun_out/a31_smoke.txt
( time timeout 900 python bench.py > gpurun_out/a31_bench.json ) 2> gpurun_out/a31_bench.err; echo EXIT=$? >> gpurun_out/a31_bench.err
( time timeout 600 python bench.py --impl reference > gpurun_out/a31_ref.json ) 2> gpurun_out/a31_ref.err; echo EXIT=$? >> gpurun_out/a31_ref.err
echo done
