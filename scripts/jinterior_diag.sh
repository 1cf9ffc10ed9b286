# Jacobi: interior blocks without boundary selects (CC_JACOBI_INTERIOR_FAST=1, default) vs 0
mkdir -p gpurun_out/ji build
make -s all > gpurun_out/ji/build.log 2>&1 || tail -20 gpurun_out/ji/build.log
lib=build/libctaclust_jnofast.so
make -s LIB=$lib PTXLOG=gpurun_out/ji/ptx.log CC_DEFS="-DCC_JACOBI_INTERIOR_FAST=0" $lib > gpurun_out/ji/build_nofast.log 2>&1
timeout -k 10 600 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_halo.py -q -x -k "jacobi or stencil or halo" --timeout 300 > gpurun_out/ji/t.log 2>&1; echo t=$?; tail -1 gpurun_out/ji/t.log
for name in fast nofast fast2 nofast2; do
  l=paper_conf_asplos_lis0l0c17_b200/libctaclust.so; case $name in nofast*) l=$lib;; esac
  CTACLUST_LIB=$PWD/$l timeout 600 python bench_suite.py gpurun_out/ji/suite_$name.json --only jacobi --quick --variants 'agent-row$|identity$|static-row-m|l2last|agent-tile8x8$' > gpurun_out/ji/suite_$name.log 2>&1
  echo "== $name rc=$?"; sed -i '/Warn\|Acsr/d' gpurun_out/ji/suite_$name.log
done
