mkdir -p gpurun_out/r10h
make all > gpurun_out/r10h/build.log 2>&1 || tail -20 gpurun_out/r10h/build.log
bash scripts/ncu_full.sh r10h conv3_tbc1:"--kernel conv3 --backend tbcluster --cluster 1" conv3_tbc2:"--kernel conv3 --backend tbcluster --cluster 2" conv3_id:"--kernel conv3 --backend identity" conv7_id:"--kernel conv7 --backend identity" conv7_st7:"--kernel conv7 --backend static --order row --clusters 1036" > gpurun_out/r10h/ncu.log 2>&1
timeout -k 10 600 python -m pytest tests/test_gpu_halo.py tests/test_gpu_runtime.py -q --timeout 400 > gpurun_out/r10h/t.log 2>&1; echo t=$?
bash scripts/sanitize.sh gpurun_out/r10h/san > gpurun_out/r10h/san.txt 2>&1
tail -3 gpurun_out/r10h/t.log; cat gpurun_out/r10h/san.txt
