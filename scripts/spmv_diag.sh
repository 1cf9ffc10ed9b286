# Diagnostic: SpMV agent knobs (L2 prefetch of the task's col/val runs, agents per SM)
mkdir -p gpurun_out/spmvd build
make -s all > gpurun_out/spmvd/build.log 2>&1
for v in "base:" "nopf:-DCC_SPMV_PREFETCH=0" "a6:-DCC_SPMV_MIN_AGENTS=6" "a6nopf:-DCC_SPMV_MIN_AGENTS=6 -DCC_SPMV_PREFETCH=0" "a4:-DCC_SPMV_MIN_AGENTS=4"; do
  name=${v%%:*}; defs=${v#*:}
  lib=paper_conf_asplos_lis0l0c17_b200/libctaclust.so
  if [ -n "$defs" ]; then
    lib=build/libctaclust_$name.so
    make -s LIB=$lib PTXLOG=gpurun_out/spmvd/ptx_$name.log CC_DEFS="$defs" $lib > gpurun_out/spmvd/build_$name.log 2>&1 || tail -5 gpurun_out/spmvd/build_$name.log
  fi
  CTACLUST_LIB=$PWD/$lib timeout 900 python bench_suite.py gpurun_out/spmvd/suite_$name.json --only spmv --variants 'agent-row$|identity$|agent-row-s|agent-row-b' > gpurun_out/spmvd/suite_$name.log 2>&1
  echo "== $name rc=$?"; sed -i '/Warn\|Acsr/d' gpurun_out/spmvd/suite_$name.log
done
