mkdir -p gpurun_out/r10e
make all > gpurun_out/r10e/build.log 2>&1 || tail -20 gpurun_out/r10e/build.log
bash scripts/ncu_full.sh r10e conv3_tbc1:"--kernel conv3 --backend tbcluster --cluster 1" conv3_tbc2:"--kernel conv3 --backend tbcluster --cluster 2" conv3_def:"--kernel conv3 --backend default" conv3_id:"--kernel conv3 --backend identity" > gpurun_out/r10e/ncu.log 2>&1
timeout -k 10 900 python -m pytest tests/test_gpu_runtime.py -q --timeout 400 > gpurun_out/r10e/t_rt.log 2>&1; echo rt=$?
tail -2 gpurun_out/r10e/t_rt.log
