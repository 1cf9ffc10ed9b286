# Diagnostic: conv 7x7 agents per SM (CC_CONV7_MIN_AGENTS) and ring depth
mkdir -p gpurun_out/c7 build
make -s all > gpurun_out/c7/build.log 2>&1
for v in "base:" "a5:-DCC_CONV7_MIN_AGENTS=5" "a7:-DCC_CONV7_MIN_AGENTS=7" "a8:-DCC_CONV7_MIN_AGENTS=8"; do
  name=${v%%:*}; defs=${v#*:}
  lib=paper_conf_asplos_lis0l0c17_b200/libctaclust.so
  if [ -n "$defs" ]; then
    lib=build/libctaclust_$name.so
    make -s LIB=$lib PTXLOG=gpurun_out/c7/ptx_$name.log CC_DEFS="$defs" $lib > gpurun_out/c7/build_$name.log 2>&1 || tail -5 gpurun_out/c7/build_$name.log
    python scripts/ptxas_regs.py gpurun_out/c7/ptx_$name.log | grep 'k_agent<cc::Conv2dBody<3>'
  fi
  CTACLUST_LIB=$PWD/$lib timeout 900 python bench_suite.py gpurun_out/c7/suite_$name.json --only conv --variants 'agent-row|identity$|agent-tile8x8-s' > gpurun_out/c7/suite_$name.log 2>&1
  echo "== $name rc=$?"; sed -i '/Warn\|Acsr/d' gpurun_out/c7/suite_$name.log
done
