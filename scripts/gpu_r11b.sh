mkdir -p gpurun_out/r11b
make all > gpurun_out/r11b/build.log 2>&1 || tail -20 gpurun_out/r11b/build.log
timeout -k 10 1500 python -m pytest tests/test_gpu_sharded.py -q --timeout 600 > gpurun_out/r11b/t.log 2>&1; echo t=$?
for c in atax jacobi conv3 conv7 spmv; do timeout -k 10 900 python bench.py --config $c > gpurun_out/r11b/bench_$c.log 2>&1; echo bench_$c=$?; done
timeout -k 10 600 python bench.py --config jacobi --fuse 1 --no-cpu-baseline --no-e2e > gpurun_out/r11b/bench_jacobi_fuse1.log 2>&1; echo bj1=$?
timeout -k 10 600 python bench.py --config jacobi --fuse 2 --no-cpu-baseline --no-e2e > gpurun_out/r11b/bench_jacobi_fuse2.log 2>&1; echo bj2=$?
timeout -k 10 600 python bench.py --impl reference --steps 3 > gpurun_out/r11b/ref_atax.log 2>&1; echo ref=$?
tail -3 gpurun_out/r11b/t.log; grep -E "^FAILED" gpurun_out/r11b/t.log | head
