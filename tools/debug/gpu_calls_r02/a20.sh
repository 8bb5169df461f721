# call 20: N>1 dry runs after the pipeline changes (short first capture round, short last HOST restore round) (every rank on GPU 0; functional, not a measurement)
mkdir -p gpurun_out
export JITC_BENCH_SHARE_GPU=1
R="python -m torch.distributed.run --nnodes=1 --master-addr 127.0.0.1"
timeout 900 $R --nproc-per-node 8 --master-port 29551 bench.py --gpus 8 --config C5 --clip 100000 --steps 3 --warmup 3 \
  --no-cpu-baseline --staging 512 --slot 128 --no-calibrate > gpurun_out/a20_c5_n8_ipc.json 2> gpurun_out/a20_c5_n8_ipc.err; echo EXIT=$? >> gpurun_out/a20_c5_n8_ipc.err
timeout 900 $R --nproc-per-node 8 --master-port 29552 bench.py --gpus 8 --config C4 --clip 100000 --steps 3 --warmup 3 \
  --no-cpu-baseline --staging 512 --slot 128 --no-calibrate > gpurun_out/a20_c4_n8_ipc.json 2> gpurun_out/a20_c4_n8_ipc.err; echo EXIT=$? >> gpurun_out/a20_c4_n8_ipc.err
timeout 900 $R --nproc-per-node 4 --master-port 29553 bench.py --gpus 4 --config C1 --steps 3 --warmup 3 \
  --no-cpu-baseline --staging 512 --slot 128 --no-calibrate --transport nccl > gpurun_out/a20_c1_n4_nccl.json 2> gpurun_out/a20_c1_n4_nccl.err; echo EXIT=$? >> gpurun_out/a20_c1_n4_nccl.err
timeout 900 $R --nproc-per-node 2 --master-port 29554 bench.py --gpus 2 --config C2 --steps 3 --warmup 3 \
  --no-cpu-baseline --hang-ctas 0 > gpurun_out/a20_c2_n2_ipc.json 2> gpurun_out/a20_c2_n2_ipc.err; echo EXIT=$? >> gpurun_out/a20_c2_n2_ipc.err
unset JITC_BENCH_SHARE_GPU

export JITC_BENCH_SHARE_GPU=1
timeout 900 python -m torch.distributed.run --nnodes=1 --master-addr 127.0.0.1 --nproc-per-node 2 --master-port 29555 bench.py --gpus 2 --config C2 --steps 3 --warmup 3 \
  --no-cpu-baseline --hang-ctas 0 --transport nccl --staging 8192 --slot 4096 > gpurun_out/a20_c2_n2_nccl.json 2> gpurun_out/a20_c2_n2_nccl.err; echo EXIT=$? >> gpurun_out/a20_c2_n2_nccl.err
echo done2
