mkdir -p gpurun_out/head
make all > gpurun_out/head/build.log 2>&1 || tail -20 gpurun_out/head/build.log
timeout -k 10 1500 python -m pytest tests/ -m gpu -q --timeout 600 -x > gpurun_out/head/t_gpu.log 2>&1; echo gpu=$?
timeout -k 10 300 python __graft_entry__.py > gpurun_out/head/smoke.log 2>&1; echo smoke=$?
timeout -k 10 600 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/head/bench.log 2>&1; echo bench=$?
timeout -k 10 600 python bench.py --config jacobi > gpurun_out/head/bench_jacobi.log 2>&1; echo bench_j=$?
tail -3 gpurun_out/head/t_gpu.log; tail -2 gpurun_out/head/smoke.log
