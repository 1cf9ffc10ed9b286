# Merged slots of up to 4 horizontally adjacent tiles (CC_STENCIL_MERGE=4) vs 2, same box
mkdir -p gpurun_out/m4 build
make -s all > gpurun_out/m4/build.log 2>&1 || tail -20 gpurun_out/m4/build.log
lib=build/libctaclust_m4.so
make -s LIB=$lib PTXLOG=gpurun_out/m4/ptx_m4.log CC_DEFS="-DCC_STENCIL_MERGE=4" $lib > gpurun_out/m4/build_m4.log 2>&1 || tail -5 gpurun_out/m4/build_m4.log
timeout -k 10 600 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_runtime.py -q -x -k "jacobi or conv or stencil or census" --timeout 300 > gpurun_out/m4/t_m2.log 2>&1; echo t_m2=$?; tail -1 gpurun_out/m4/t_m2.log
CTACLUST_LIB=$PWD/$lib timeout -k 10 600 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_runtime.py -q -x -k "jacobi or conv or stencil or census" --timeout 300 > gpurun_out/m4/t_m4.log 2>&1; echo t_m4=$?; tail -3 gpurun_out/m4/t_m4.log
for name in m2 m4 m2b m4b; do
  l=paper_conf_asplos_lis0l0c17_b200/libctaclust.so; case $name in m4*) l=$lib;; esac
  CTACLUST_LIB=$PWD/$l timeout 600 python scripts/vpair_probe.py > gpurun_out/m4/probe_$name.log 2>&1
  CTACLUST_LIB=$PWD/$l timeout 900 python bench_suite.py gpurun_out/m4/suite_$name.json --only jacobi,conv --variants 'agent-row$|identity$|agent-tile8x8$|static-row|l2last' > gpurun_out/m4/suite_$name.log 2>&1
  echo "== $name rc=$?"; sed -i '/Warn\|Acsr/d' gpurun_out/m4/suite_$name.log gpurun_out/m4/probe_$name.log
done
