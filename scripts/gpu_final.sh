# final pass: GPU suite, smoke, bench every config (default flags), reference arm, bench launch list + ncu captures
mkdir -p gpurun_out/final
make all > gpurun_out/final/build.log 2>&1 || tail -20 gpurun_out/final/build.log
timeout -k 10 2400 python -m pytest tests/ -m gpu -q --timeout 900 > gpurun_out/final/t_gpu.log 2>&1; echo gpu=$?
timeout -k 10 300 python __graft_entry__.py > gpurun_out/final/smoke.log 2>&1; echo smoke=$?
timeout -k 10 900 python bench.py --gpus 1 --steps 20 --warmup 5 > gpurun_out/final/bench_driver_cmd.log 2>&1; echo bench=$?
for c in atax jacobi conv3 conv7 spmv; do timeout -k 10 900 python bench.py --config $c > gpurun_out/final/bench_$c.log 2>&1; echo bench_$c=$?; done
timeout -k 10 600 python bench.py --impl reference --gpus 1 --steps 20 --warmup 5 > gpurun_out/final/ref.log 2>&1; echo ref=$?
bash scripts/ncu_bench.sh final > gpurun_out/final/ncu_bench.log 2>&1
tail -3 gpurun_out/final/t_gpu.log; grep -E "^FAILED" gpurun_out/final/t_gpu.log | head; tail -2 gpurun_out/final/smoke.log
