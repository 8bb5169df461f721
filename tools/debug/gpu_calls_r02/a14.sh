# call 14: new segment-boundary parity test (128 KiB segments x 64 KiB / 1 MiB chunks x misalignment)
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "segment_boundaries" > gpurun_out/a14_seg_tests.txt 2>&1; echo EXIT=$? >> gpurun_out/a14_seg_tests.txt
echo done
