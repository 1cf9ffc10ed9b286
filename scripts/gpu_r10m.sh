mkdir -p gpurun_out/r10m
make all > gpurun_out/r10m/build.log 2>&1 || tail -20 gpurun_out/r10m/build.log
timeout -k 10 1200 python -m pytest tests/test_gpu_sharded.py tests/test_gpu_kernels.py -q --timeout 600 -k "sharded or bench or spmv or window" > gpurun_out/r10m/t.log 2>&1; echo t=$?
timeout -k 10 900 python bench.py --config spmv > gpurun_out/r10m/bench_spmv.log 2>&1; echo b=$?
tail -5 gpurun_out/r10m/t.log; grep -E "^FAILED" gpurun_out/r10m/t.log | head; tail -c 1500 gpurun_out/r10m/bench_spmv.log
