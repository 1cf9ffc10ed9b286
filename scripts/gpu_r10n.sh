mkdir -p gpurun_out/r10n
make all > gpurun_out/r10n/build.log 2>&1 || tail -20 gpurun_out/r10n/build.log
timeout -k 10 1500 python -m pytest tests/test_gpu_sharded.py -q --timeout 600 > gpurun_out/r10n/t.log 2>&1; echo t=$?
tail -5 gpurun_out/r10n/t.log; grep -E "^FAILED" gpurun_out/r10n/t.log | head
