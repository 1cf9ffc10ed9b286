mkdir -p gpurun_out/r10c
make all > gpurun_out/r10c/build.log 2>&1 || tail -20 gpurun_out/r10c/build.log
timeout -k 10 900 python -m pytest tests/test_gpu_sharded.py tests/test_gpu_kernels.py -q -x --timeout 400 -k "sharded or window or driver or spmv" > gpurun_out/r10c/t.log 2>&1; echo t=$?
timeout -k 10 900 python scripts/exp_r10.py spmv gpurun_out/r10c/spmv.json > gpurun_out/r10c/spmv.log 2>&1; echo spmv=$?
timeout -k 10 900 python scripts/exp_r10.py stencil gpurun_out/r10c/stencil.json > gpurun_out/r10c/stencil.log 2>&1; echo st=$?
for c in conv3 spmv; do timeout -k 10 600 python bench.py --config $c --no-cpu-baseline > gpurun_out/r10c/bench_$c.log 2>&1; echo bench_$c=$?; done
tail -2 gpurun_out/r10c/t.log; cat gpurun_out/r10c/spmv.log gpurun_out/r10c/stencil.log | cut -c1-1500
