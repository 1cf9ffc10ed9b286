# Diagnostic: consumer groups per conv agent (1 = one producer warp per group).
mkdir -p gpurun_out build
make -s all > gpurun_out/build.log 2>&1
for v in "g0:" "g1:-DCC_CONV_GROUPS=1" "g2:-DCC_CONV_GROUPS=2"; do
  name=${v%%:*}; defs=${v#*:}
  lib=paper_conf_asplos_lis0l0c17_b200/libctaclust.so
  if [ -n "$defs" ]; then
    lib=build/libctaclust_$name.so
    make -s LIB=$lib PTXLOG=gpurun_out/ptx_$name.log CC_DEFS="$defs" $lib > gpurun_out/build_$name.log 2>&1 || tail -5 gpurun_out/build_$name.log
  fi
  CTACLUST_LIB=$PWD/$lib timeout 1200 python bench_suite.py gpurun_out/suite_g_$name.json --only conv --quick > gpurun_out/suite_g_$name.log 2>&1
  echo "== $name rc=$?"
done
