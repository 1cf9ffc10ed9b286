# Diagnostic: ring waits as test_wait + timed nanosleep (producer / consumer
# maximum back-off in ns) vs the suspend-hint try_wait.  CTACLUST_LIB selects.
mkdir -p gpurun_out/sleep build
make -s all > gpurun_out/sleep/build.log 2>&1
for v in "base:" "p512:-DCC_PROD_SLEEP=512" "p512c128:-DCC_PROD_SLEEP=512 -DCC_CONS_SLEEP=128" \
         "p2048c256:-DCC_PROD_SLEEP=2048 -DCC_CONS_SLEEP=256" "p256c64:-DCC_PROD_SLEEP=256 -DCC_CONS_SLEEP=64"; do
  name=${v%%:*}; defs=${v#*:}
  lib=paper_conf_asplos_lis0l0c17_b200/libctaclust.so
  if [ -n "$defs" ]; then
    lib=build/libctaclust_$name.so
    make -s LIB=$lib PTXLOG=gpurun_out/sleep/ptx_$name.log CC_DEFS="$defs" $lib > gpurun_out/sleep/build_$name.log 2>&1 || tail -5 gpurun_out/sleep/build_$name.log
  fi
  CTACLUST_LIB=$PWD/$lib timeout 900 python bench_suite.py gpurun_out/sleep/suite_$name.json --quick --only atax,jacobi,conv,spmv,hist \
     --variants 'agent-row$|agent-col$|identity$' > gpurun_out/sleep/suite_$name.log 2>&1
  echo "== $name rc=$?"
  sed -i '/Warn\|Acsr/d' gpurun_out/sleep/suite_$name.log
done
