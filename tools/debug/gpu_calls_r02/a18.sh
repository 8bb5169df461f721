# call 18: capture as one pipeline across groups with a short first round: GPU suite, C3 bench, timeline
mkdir -p gpurun_out
( time timeout 1800 python -m pytest tests -m gpu -x -q ) > gpurun_out/a18_gpu_tests.txt 2>&1; echo EXIT=$? >> gpurun_out/a18_gpu_tests.txt
timeout 900 python bench.py > gpurun_out/a18_bench.json 2> gpurun_out/a18_bench.err; echo EXIT=$? >> gpurun_out/a18_bench.err
timeout 900 python tools/timeline.py --config C3 --out gpurun_out/a18_timeline_c3 > gpurun_out/a18_timeline.log 2>&1; echo EXIT=$? >> gpurun_out/a18_timeline.log
echo done
