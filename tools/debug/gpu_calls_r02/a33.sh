# call 33: K5 fused peer pull with the round-2 kernel shapes (C2 and C3; writer and replacement on one GPU)
mkdir -p gpurun_out
timeout 900 python tools/pull_bench.py C2 3 > gpurun_out/a33_pull_c2.json 2> gpurun_out/a33_pull_c2.err; echo EXIT=$? >> gpurun_out/a33_pull_c2.err
echo done
