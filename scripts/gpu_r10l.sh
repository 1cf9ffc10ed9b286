mkdir -p gpurun_out/r10l
L=paper_conf_asplos_lis0l0c17_b200
make all > gpurun_out/r10l/build.log 2>&1 || tail -20 gpurun_out/r10l/build.log
make LIB=$L/lib_xcg.so CC_DEFS="-DCC_SPMV_XCG=1" PTXLOG=/tmp/p_xcg.log > /dev/null 2>&1
echo "== base"; EXP_SPMV_HOTS=0,16384 timeout -k 10 900 python scripts/exp_r10.py spmv gpurun_out/r10l/spmv_base.json 2>&1 | head -3 | cut -c1-400
echo "== xcg"; EXP_SPMV_HOTS=0,16384 CTACLUST_LIB=$PWD/$L/lib_xcg.so timeout -k 10 900 python scripts/exp_r10.py spmv gpurun_out/r10l/spmv_xcg.json 2>&1 | head -3 | cut -c1-400
bash scripts/ncu_full.sh r10l conv7_tbc1:"--kernel conv7 --backend tbcluster --cluster 1"; CTACLUST_LIB=$PWD/$L/lib_xcg.so bash scripts/ncu_full.sh r10l spmv_xcg_def:"--kernel spmv --backend default" > gpurun_out/r10l/ncu.log 2>&1
