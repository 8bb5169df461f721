# call 21: PEER plans end with a short round too: multi-rank / PEER GPU tests + C2 N=2 IPC dry run
mkdir -p gpurun_out
( time timeout 1500 python -m pytest tests/test_gpu_multirank.py tests/test_gpu_peer_pull.py tests/test_gpu_scenarios.py tests/test_gpu_bench_multirank.py tests/test_gpu_writer_death.py tests/test_gpu_fanout.py -q ) > gpurun_out/a21_tests.txt 2>&1; echo EXIT=$? >> gpurun_out/a21_tests.txt
JITC_BENCH_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --master-addr 127.0.0.1 --nproc-per-node 2 --master-port 29561 bench.py --gpus 2 --config C2 --steps 3 --warmup 3 \
  --no-cpu-baseline --hang-ctas 0 > gpurun_out/a21_c2_n2_ipc.json 2> gpurun_out/a21_c2_n2_ipc.err; echo EXIT=$? >> gpurun_out/a21_c2_n2_ipc.err
echo done
