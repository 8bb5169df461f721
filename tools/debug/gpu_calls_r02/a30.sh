# call 30: fan-out capture plans visit the lanes round-robin: fan-out GPU tests + C5 / C4 8-rank dry runs (fan-out default)
mkdir -p gpurun_out
( time timeout 1500 python -m pytest tests/test_gpu_fanout.py tests/test_gpu_scenarios.py -q ) > gpurun_out/a30_tests.txt 2>&1; echo EXIT=$? >> gpurun_out/a30_tests.txt
export JITC_BENCH_SHARE_GPU=1
R="python -m torch.distributed.run --nnodes=1 --master-addr 127.0.0.1"
timeout 900 $R --nproc-per-node 8 --master-port 29571 bench.py --gpus 8 --config C5 --clip 100000 --steps 3 --warmup 3 \
  --no-cpu-baseline --staging 512 --slot 128 --no-calibrate > gpurun_out/a30_c5_n8_ipc.json 2> gpurun_out/a30_c5_n8_ipc.err; echo EXIT=$? >> gpurun_out/a30_c5_n8_ipc.err
timeout 900 $R --nproc-per-node 8 --master-port 29572 bench.py --gpus 8 --config C4 --clip 100000 --steps 3 --warmup 3 \
  --no-cpu-baseline --staging 512 --slot 128 --no-calibrate > gpurun_out/a30_c4_n8_ipc.json 2> gpurun_out/a30_c4_n8_ipc.err; echo EXIT=$? >> gpurun_out/a30_c4_n8_ipc.err
timeout 900 $R --nproc-per-node 8 --master-port 29573 bench.py --gpus 8 --config C5 --clip 30000 --steps 3 --warmup 3 \
  --no-cpu-baseline --staging 512 --slot 128 --no-calibrate --transport nccl > gpurun_out/a30_c5_n8_nccl.json 2> gpurun_out/a30_c5_n8_nccl.err; echo EXIT=$? >> gpurun_out/a30_c5_n8_nccl.err
echo done
