# conv 3x3: one consumer group per agent with more agents per SM (a producer warp per group) vs 2 groups x 4 agents
mkdir -p gpurun_out/sa build
make -s all > gpurun_out/sa/build.log 2>&1
for v in "g1a8:-DCC_CONV_GROUPS=1 -DCC_CONV3_MIN_AGENTS=8" "g1a7:-DCC_CONV_GROUPS=1 -DCC_CONV3_MIN_AGENTS=7" "g1a6:-DCC_CONV_GROUPS=1 -DCC_CONV3_MIN_AGENTS=6"; do
  name=${v%%:*}; defs=${v#*:}
  make -s LIB=build/libctaclust_$name.so PTXLOG=gpurun_out/sa/ptx_$name.log CC_DEFS="$defs" build/libctaclust_$name.so > gpurun_out/sa/build_$name.log 2>&1 || tail -5 gpurun_out/sa/build_$name.log
  python scripts/ptxas_regs.py gpurun_out/sa/ptx_$name.log | grep 'k_agent<cc::Conv2dBody<1>'
done
for name in base g1a8 g1a7 g1a6 base2; do
  l=paper_conf_asplos_lis0l0c17_b200/libctaclust.so; case $name in g1*) l=build/libctaclust_$name.so;; esac
  CTACLUST_LIB=$PWD/$l timeout 600 python bench_suite.py gpurun_out/sa/suite_$name.json --only conv --variants 'agent-row$|identity$|agent-row-l2last' > gpurun_out/sa/suite_$name.log 2>&1
  echo "== $name rc=$?"; sed -i '/Warn\|Acsr/d' gpurun_out/sa/suite_$name.log
done
