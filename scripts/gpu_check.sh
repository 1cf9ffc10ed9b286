# GPU correctness + bench pass (run under gpurun from the repo root)
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
make all > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
timeout -k 10 300 python __graft_entry__.py > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout -k 10 600 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_comm.py tests/test_gpu_halo.py tests/test_gpu_categorize.py tests/test_gpu_microbench.py -q --timeout 300 > gpurun_out/t_runtime.log 2>&1; echo rt=$?
timeout -k 10 1500 python -m pytest tests/test_gpu_kernels.py -q --timeout 400 > gpurun_out/t_kernels.log 2>&1; echo k=$?
timeout -k 10 600 python bench.py --steps 100 --warmup 5 > gpurun_out/bench.log 2>&1; echo b=$?
timeout -k 10 1200 python bench_suite.py gpurun_out/suite.json ${SUITE_ARGS} > gpurun_out/suite.log 2>&1; echo s=$?
for f in smoke t_runtime t_kernels bench; do echo "== $f"; tail -n 4 gpurun_out/$f.log; done
