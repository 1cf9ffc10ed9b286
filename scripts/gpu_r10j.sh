# TB-cluster pair layout (parity + perf), SpMV controls (permuted R-MAT, inspector USER order), agent L2 prefetch A/B
mkdir -p gpurun_out/r10j
L=paper_conf_asplos_lis0l0c17_b200
make all > gpurun_out/r10j/build.log 2>&1 || tail -20 gpurun_out/r10j/build.log
make LIB=$L/lib_nopf.so CC_DEFS="-DCC_SPMV_PREFETCH=0" PTXLOG=/tmp/p_nopf.log > /dev/null 2>&1 &
for ns in 250 500 1000 2000; do make LIB=$L/lib_c7p$ns.so CC_DEFS="-DCC_CONV7_PROD_NS=$ns" PTXLOG=/tmp/p_c7p$ns.log > /dev/null 2>&1 & done
timeout -k 10 600 python -m pytest tests/test_gpu_kernels.py -q -x --timeout 400 -k "tbc or conv" > gpurun_out/r10j/t_conv.log 2>&1; echo tconv=$?
timeout -k 10 600 python scripts/sanitize_targets.py tbc > gpurun_out/r10j/san_tbc_plain.log 2>&1; echo santbc=$?
timeout -k 10 600 compute-sanitizer --tool racecheck --error-exitcode 9 python scripts/sanitize_targets.py tbc > gpurun_out/r10j/racecheck_tbc.log 2>&1; echo race_tbc=$?
timeout -k 10 600 compute-sanitizer --tool synccheck --error-exitcode 9 python scripts/sanitize_targets.py tbc > gpurun_out/r10j/synccheck_tbc.log 2>&1; echo sync_tbc=$?
timeout -k 10 600 python scripts/exp_r10.py tbc gpurun_out/r10j/tbc.json > gpurun_out/r10j/tbc.log 2>&1; echo tbc=$?
bash scripts/ncu_full.sh r10j conv3_tbc2:"--kernel conv3 --backend tbcluster --cluster 2" > gpurun_out/r10j/ncu.log 2>&1
timeout -k 10 900 python scripts/exp_r10.py spmv_control gpurun_out/r10j/spmv_control.json > gpurun_out/r10j/spmv_control.log 2>&1; echo spc=$?
wait
echo "== base"; EXP_SPMV_HOTS=0 timeout -k 10 900 python scripts/exp_r10.py spmv gpurun_out/r10j/spmv_base.json 2>&1 | head -3 | cut -c1-400
echo "== nopf"; EXP_SPMV_HOTS=0 CTACLUST_LIB=$PWD/$L/lib_nopf.so timeout -k 10 900 python scripts/exp_r10.py spmv gpurun_out/r10j/spmv_nopf.json 2>&1 | head -3 | cut -c1-400
echo "== c7 base"; timeout -k 10 300 python scripts/exp_r10.py conv7 gpurun_out/r10j/c7_base.json 2>&1 | cut -c1-900
for ns in 250 500 1000 2000; do echo "== c7 prod sleep $ns"; CTACLUST_LIB=$PWD/$L/lib_c7p$ns.so timeout -k 10 300 python scripts/exp_r10.py conv7 gpurun_out/r10j/c7_p$ns.json 2>&1 | cut -c1-900; done
tail -2 gpurun_out/r10j/t_conv.log; tail -2 gpurun_out/r10j/racecheck_tbc.log gpurun_out/r10j/synccheck_tbc.log; cat gpurun_out/r10j/tbc.log gpurun_out/r10j/spmv_control.log | cut -c1-900
