mkdir -p gpurun_out/r10d
make all > gpurun_out/r10d/build.log 2>&1 || tail -20 gpurun_out/r10d/build.log
make LIB=paper_conf_asplos_lis0l0c17_b200/libctaclust_ctascope.so CC_DEFS="-DCC_TBC_CTA_SCOPE=1" PTXLOG=/tmp/p.log > /dev/null 2>&1
timeout -k 10 600 python -m pytest tests/test_gpu_kernels.py -q -x --timeout 400 -k "tbc or conv" > gpurun_out/r10d/t_conv.log 2>&1; echo tconv=$?
timeout -k 10 600 python -m pytest tests/test_gpu_sharded.py -q --timeout 400 -k "ranks" > gpurun_out/r10d/t_sh.log 2>&1; echo tsh=$?
timeout -k 10 600 python scripts/exp_r10.py tbc gpurun_out/r10d/tbc.json > gpurun_out/r10d/tbc.log 2>&1; echo tbc=$?
CTACLUST_LIB=$PWD/paper_conf_asplos_lis0l0c17_b200/libctaclust_ctascope.so timeout -k 10 600 python scripts/exp_r10.py tbc gpurun_out/r10d/tbc_cta.json > gpurun_out/r10d/tbc_cta.log 2>&1; echo tbc2=$?
timeout -k 10 600 python scripts/exp_r10.py panel gpurun_out/r10d/panel.json > gpurun_out/r10d/panel.log 2>&1; echo panel=$?
tail -2 gpurun_out/r10d/t_conv.log gpurun_out/r10d/t_sh.log; cat gpurun_out/r10d/tbc.log gpurun_out/r10d/tbc_cta.log gpurun_out/r10d/panel.log | cut -c1-1200
