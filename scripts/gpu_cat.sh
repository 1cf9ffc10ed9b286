mkdir -p gpurun_out
make all > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
timeout -k 10 900 python -m pytest tests -m gpu -q --timeout 400 -x > gpurun_out/t_gpu_all.log 2>&1; echo "tests=$?"; tail -3 gpurun_out/t_gpu_all.log
timeout -k 10 1800 python scripts/categorize_run.py gpurun_out/categorize.json > gpurun_out/categorize.log 2>&1; echo "cat=$?"; tail -12 gpurun_out/categorize.log
