# call 15: N>1 dry runs of bench.py with the round-2 kernel shapes (every rank on GPU 0; functional, not a measurement)
mkdir -p gpurun_out
export JITC_BENCH_SHARE_GPU=1
R="python -m torch.distributed.run --nnodes=1 --master-addr 127.0.0.1"
timeout 900 $R --nproc-per-node 8 --master-port 29541 bench.py --gpus 8 --config C5 --clip 100000 --steps 3 --warmup 3 \
  --no-cpu-baseline --staging 512 --slot 128 --no-calibrate > gpurun_out/a15_c5_n8_ipc.json 2> gpurun_out/a15_c5_n8_ipc.err; echo EXIT=$? >> gpurun_out/a15_c5_n8_ipc.err
timeout 900 $R --nproc-per-node 8 --master-port 29542 bench.py --gpus 8 --config C4 --clip 100000 --steps 3 --warmup 3 \
  --no-cpu-baseline --staging 512 --slot 128 --no-calibrate > gpurun_out/a15_c4_n8_ipc.json 2> gpurun_out/a15_c4_n8_ipc.err; echo EXIT=$? >> gpurun_out/a15_c4_n8_ipc.err
timeout 900 $R --nproc-per-node 4 --master-port 29543 bench.py --gpus 4 --config C1 --steps 3 --warmup 3 \
  --no-cpu-baseline --staging 512 --slot 128 --no-calibrate --transport nccl > gpurun_out/a15_c1_n4_nccl.json 2> gpurun_out/a15_c1_n4_nccl.err; echo EXIT=$? >> gpurun_out/a15_c1_n4_nccl.err
timeout 900 $R --nproc-per-node 2 --master-port 29544 bench.py --gpus 2 --config C2 --steps 3 --warmup 3 \
  --no-cpu-baseline --hang-ctas 0 > gpurun_out/a15_c2_n2_ipc.json 2> gpurun_out/a15_c2_n2_ipc.err; echo EXIT=$? >> gpurun_out/a15_c2_n2_ipc.err
unset JITC_BENCH_SHARE_GPU
timeout 600 python bench.py --impl reference > gpurun_out/a15_ref.json 2> gpurun_out/a15_ref.err; echo EXIT=$? >> gpurun_out/a15_ref.err
echo done
