# Diagnostic: cost of the fused LL halo per slab sweep kernel (launch list of
# fused vs plain kernels) for the shipped build and diagnostic builds.
mkdir -p gpurun_out build
make -s all > gpurun_out/build.log 2>&1
for v in ${LL_VARIANTS:-"sys:"}; do
  name=${v%%:*}; defs=${v#*:}
  lib=paper_conf_asplos_lis0l0c17_b200/libctaclust.so
  if [ -n "$defs" ]; then
    lib=build/libctaclust_$name.so
    make -s LIB=$lib PTXLOG=gpurun_out/ptx_$name.log CC_DEFS="$defs" $lib > gpurun_out/build_$name.log 2>&1 || tail -5 gpurun_out/build_$name.log
  fi
  CTACLUST_LIB=$PWD/$lib timeout -k 10 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv \
     --log-file gpurun_out/ll_$name.csv python scripts/slab_ncu.py ${SLAB_ARGS} > gpurun_out/ll_$name.log 2>&1
  echo "== $name rc=$?"
  python scripts/launch_csv.py gpurun_out/ll_$name.csv Jacobi
done
