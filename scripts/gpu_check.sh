mkdir -p gpurun_out
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
make all > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
timeout -k 10 300 python __graft_entry__.py > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout -k 10 600 python -m pytest tests/test_gpu_runtime.py -x -q --timeout 120 > gpurun_out/t_runtime.log 2>&1; echo rt=$?
timeout -k 10 1200 python -m pytest tests/test_gpu_kernels.py -q --timeout 300 -x > gpurun_out/t_kernels.log 2>&1; echo k=$?
timeout -k 10 600 python bench.py --steps 100 --warmup 5 > gpurun_out/bench.log 2>&1; echo b=$?
tail -3 gpurun_out/smoke.log gpurun_out/t_runtime.log gpurun_out/t_kernels.log gpurun_out/bench.log
