mkdir -p gpurun_out/r10f
make all > gpurun_out/r10f/build.log 2>&1 || tail -20 gpurun_out/r10f/build.log
timeout -k 10 600 python -m pytest tests/test_gpu_kernels.py -q -x --timeout 400 -k "tbc or conv" > gpurun_out/r10f/t_conv.log 2>&1; echo tconv=$?
timeout -k 10 600 python scripts/exp_r10.py tbc gpurun_out/r10f/tbc.json > gpurun_out/r10f/tbc.log 2>&1; echo tbc=$?
bash scripts/ncu_full.sh r10f conv3_tbc2:"--kernel conv3 --backend tbcluster --cluster 2" > gpurun_out/r10f/ncu.log 2>&1
tail -2 gpurun_out/r10f/t_conv.log; cat gpurun_out/r10f/tbc.log | cut -c1-1200
