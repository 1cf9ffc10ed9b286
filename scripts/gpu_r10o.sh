mkdir -p gpurun_out/r10o
make all > gpurun_out/r10o/build.log 2>&1 || tail -20 gpurun_out/r10o/build.log
timeout -k 10 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_sharded.py -q --timeout 600 -k "atax or bench_two_ranks" > gpurun_out/r10o/t.log 2>&1; echo t=$?
timeout -k 10 900 python bench.py > gpurun_out/r10o/bench_atax.log 2>&1; echo b=$?
bash scripts/ncu_full.sh r10o atax_fused:"--kernel atax_fused --backend agent" > gpurun_out/r10o/ncu.log 2>&1
tail -3 gpurun_out/r10o/t.log; grep -E "^FAILED" gpurun_out/r10o/t.log | head; tail -c 2500 gpurun_out/r10o/bench_atax.log
