# call 44: TSAN stress now also runs persist / stage-in (I/O threads, bounce-buffer copier threads)
mkdir -p gpurun_out
timeout 1200 python -m pytest tests/test_tsan.py -q > gpurun_out/a44_tsan.txt 2>&1; echo EXIT=$? >> gpurun_out/a44_tsan.txt
echo done
