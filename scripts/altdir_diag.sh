# Diagnostic: odd clusters drained back to front (CC_ALT_DIR=1) vs front to back.
mkdir -p gpurun_out/alt build
make -s all > gpurun_out/alt/build.log 2>&1
lib=build/libctaclust_alt.so
make -s LIB=$lib PTXLOG=gpurun_out/alt/ptx_alt.log CC_DEFS="-DCC_ALT_DIR=1" $lib > gpurun_out/alt/build_alt.log 2>&1 || tail -5 gpurun_out/alt/build_alt.log
CTACLUST_LIB=$PWD/$lib timeout -k 10 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_runtime.py -q -x --timeout 400 > gpurun_out/alt/t_alt.log 2>&1; echo t_alt=$?; tail -2 gpurun_out/alt/t_alt.log
for name in base alt; do
  l=paper_conf_asplos_lis0l0c17_b200/libctaclust.so; [ $name = alt ] && l=$lib
  CTACLUST_LIB=$PWD/$l timeout 900 python bench_suite.py gpurun_out/alt/suite_$name.json --only atax,jacobi,conv \
     --variants 'agent-row$|agent-col$|identity$|static-row-m|agent-row-l2last' > gpurun_out/alt/suite_$name.log 2>&1
  echo "== $name rc=$?"; sed -i '/Warn\|Acsr/d' gpurun_out/alt/suite_$name.log
done
