# interleaved USER-order rows (time-aligned clusters) + USER-order parity
mkdir -p gpurun_out/exp3
make all > gpurun_out/exp3/build.log 2>&1 || tail -20 gpurun_out/exp3/build.log
timeout -k 10 600 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_runtime.py -q -x -k 'user or census or runtime' --timeout 300 > gpurun_out/exp3/t_user.log 2>&1; echo t=$?; tail -3 gpurun_out/exp3/t_user.log
timeout -k 10 900 python bench_suite.py gpurun_out/exp3/suite.json --only jacobi,conv --variants 'ilv|identity$|agent-row$' > gpurun_out/exp3/suite.log 2>&1; echo s=$?
grep -v Warn gpurun_out/exp3/suite.log | grep -v Acsr | tail -40
