timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_sharded.py -k "spmv" -x -q 2>&1 | tail -3
timeout 900 python bench.py --config spmv > gpurun_out/bench_spmv_shub.json 2> gpurun_out/bench_spmv_shub.err; tail -c 3000 gpurun_out/bench_spmv_shub.json
