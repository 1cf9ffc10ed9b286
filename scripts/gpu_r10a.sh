mkdir -p gpurun_out
make all > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
timeout -k 10 900 python -m pytest tests/ -m gpu -q -x --timeout 400 -k "jacobi or halo or slab" > gpurun_out/t_jac.log 2>&1; echo jac=$?
bash scripts/ncu_full.sh r10 spmv_def:"--kernel spmv --backend default" spmv_agent:"--kernel spmv --backend agent" > gpurun_out/ncu_full_r10.log 2>&1
tail -3 gpurun_out/t_jac.log
