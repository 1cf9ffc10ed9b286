mkdir -p gpurun_out/r12a
make all > gpurun_out/r12a/build.log 2>&1 || tail -20 gpurun_out/r12a/build.log
timeout -k 10 900 python -m pytest tests/test_gpu_kernels.py -q --timeout 600 -k "spmv" > gpurun_out/r12a/t.log 2>&1; echo t=$?
EXP_SPMV_HOTS=0,16384 timeout -k 10 900 python scripts/exp_r10.py spmv gpurun_out/r12a/spmv.json 2>&1 | cut -c1-400
bash scripts/ncu_full.sh r12a spmv_def:"--kernel spmv --backend default --hot 16384" > gpurun_out/r12a/ncu.log 2>&1
tail -2 gpurun_out/r12a/t.log
