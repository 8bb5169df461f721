# session-2 call 12: compute-sanitizer on the changed kernels and the fan-out path; C3 with the current defaults;
# C2 N=2 on one GPU (IPC, full size; functional)
mkdir -p gpurun_out
CS=/usr/local/cuda/bin/compute-sanitizer
timeout 1500 $CS --tool memcheck --leak-check no python -m pytest tests/test_gpu_parity.py -q \
  -k "k1_digests_match_oracle and 4096 or capture_restore_bit_exact and 4096 or edge or k4_" > gpurun_out/s12_memcheck_parity.log 2>&1; echo EXIT=$? >> gpurun_out/s12_memcheck_parity.log
timeout 1500 $CS --tool memcheck --leak-check no --target-processes all python -m pytest tests/test_gpu_fanout.py -q -k "ipc" > gpurun_out/s12_memcheck_fanout.log 2>&1; echo EXIT=$? >> gpurun_out/s12_memcheck_fanout.log
timeout 900 $CS --tool racecheck python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s12_racecheck.log 2>&1; echo EXIT=$? >> gpurun_out/s12_racecheck.log
timeout 900 $CS --tool synccheck python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/s12_synccheck.log 2>&1; echo EXIT=$? >> gpurun_out/s12_synccheck.log
timeout 900 python bench.py --config C3 --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/s12_bench_c3.json 2> gpurun_out/s12_bench_c3.err
JITC_BENCH_SHARE_GPU=1 timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29513 \
  bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu-baseline --hang-ctas 0 > gpurun_out/s12_bench_c2_n2share.json 2> gpurun_out/s12_bench_c2_n2share.err
echo done
