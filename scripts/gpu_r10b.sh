# round-2 check: full GPU suite + bench every config at N=1
mkdir -p gpurun_out/r10b
make all > gpurun_out/r10b/build.log 2>&1 || tail -20 gpurun_out/r10b/build.log
timeout -k 10 900 python -m pytest tests/test_gpu_sharded.py -q -x --timeout 400 > gpurun_out/r10b/t_sharded.log 2>&1; echo sharded=$?
timeout -k 10 1200 python -m pytest tests/ -m gpu -q --timeout 400 > gpurun_out/r10b/t_gpu.log 2>&1; echo gpu=$?
for c in atax jacobi conv3 conv7 spmv; do
  timeout -k 10 600 python bench.py --config $c > gpurun_out/r10b/bench_$c.log 2>&1; echo bench_$c=$?
done
tail -3 gpurun_out/r10b/t_sharded.log gpurun_out/r10b/t_gpu.log
for c in atax jacobi conv3 conv7 spmv; do tail -c 600 gpurun_out/r10b/bench_$c.log; echo; done
