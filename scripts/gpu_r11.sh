# round-2 final evidence: GPU suite, bench every config, ncu suite + bench launch list (tag r11)
mkdir -p gpurun_out/r11
make all > gpurun_out/r11/build.log 2>&1 || tail -20 gpurun_out/r11/build.log
timeout -k 10 1800 python -m pytest tests/ -m gpu -q --timeout 600 > gpurun_out/r11/t_gpu.log 2>&1; echo gpu=$?
timeout -k 10 300 python __graft_entry__.py > gpurun_out/r11/smoke.log 2>&1; echo smoke=$?
bash scripts/ncu_suite.sh r11 > gpurun_out/r11/ncu_suite.log 2>&1
bash scripts/ncu_bench.sh r11 > gpurun_out/r11/ncu_bench.log 2>&1
tail -3 gpurun_out/r11/t_gpu.log; grep -E "^FAILED" gpurun_out/r11/t_gpu.log | head; cat gpurun_out/r11/smoke.log | tail -2
