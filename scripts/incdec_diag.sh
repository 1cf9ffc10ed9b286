# Incremental order decode in the scheduler (CC_INC_DECODE=1, default) vs full Eq. 7 + Fig. 7 decode per pop
mkdir -p gpurun_out/inc3 build
make -s all > gpurun_out/inc3/build.log 2>&1 || tail -20 gpurun_out/inc3/build.log
: timeout -k 10 900 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_kernels.py -q -x --timeout 400 > gpurun_out/inc3/t.log 2>&1; echo t=$?; tail -2 gpurun_out/inc3/t.log
lib=build/libctaclust_full.so
make -s LIB=$lib PTXLOG=gpurun_out/inc3/ptx_full.log CC_DEFS="-DCC_INC_DECODE=0" $lib > gpurun_out/inc3/build_full.log 2>&1 || tail -5 gpurun_out/inc3/build_full.log
for name in full inc full2 inc2; do
  l=paper_conf_asplos_lis0l0c17_b200/libctaclust.so; case $name in full*) l=$lib;; esac
  CTACLUST_LIB=$PWD/$l timeout 900 python bench_suite.py gpurun_out/inc3/suite_$name.json --only conv \
     --variants 'agent-row$|agent-col$|identity$|agent-tile|agent-row-l2last|agent-band' > gpurun_out/inc3/suite_$name.log 2>&1
  echo "== $name rc=$?"; sed -i '/Warn\|Acsr/d' gpurun_out/inc3/suite_$name.log
done
