# Diagnostic: mbarrier wait form (suspend hint vs nanosleep backoff) on the
# stencil suites.  Builds the variants on the box; CTACLUST_LIB selects.
mkdir -p gpurun_out build
make -s all > gpurun_out/build.log 2>&1
for v in "hint:" "bo256:-DCC_WAIT_BACKOFF=256" "bo1024:-DCC_WAIT_BACKOFF=1024"; do
  name=${v%%:*}; defs=${v#*:}
  lib=paper_conf_asplos_lis0l0c17_b200/libctaclust.so
  if [ -n "$defs" ]; then
    lib=build/libctaclust_$name.so
    make -s LIB=$lib PTXLOG=gpurun_out/ptx_$name.log CC_DEFS="$defs" $lib > gpurun_out/build_$name.log 2>&1 || tail -5 gpurun_out/build_$name.log
  fi
  CTACLUST_LIB=$PWD/$lib timeout 1200 python bench_suite.py gpurun_out/suite_w_$name.json --only ${WAIT_SUITES:-conv,jacobi} --quick > gpurun_out/suite_w_$name.log 2>&1
  echo "== $name rc=$?"
done
