for i in 1 2 3; do timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_sharded.py -k "jacobi" -x -q --tb=short 2>&1 | grep -vE "^\.|^$" | tail -30 | cut -c1-600; done
