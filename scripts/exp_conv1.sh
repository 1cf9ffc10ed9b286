# conv: one tile-code instance for both staging paths (default) vs the duplicated body, same box
mkdir -p gpurun_out/c2 build
make -s all > gpurun_out/c2/build.log 2>&1 || tail -20 gpurun_out/c2/build.log
lib=build/libctaclust_dual.so
make -s LIB=$lib PTXLOG=gpurun_out/c2/ptx_dual.log CC_DEFS="-DCC_CONV_DUAL_BODY=1" $lib > gpurun_out/c2/build_dual.log 2>&1 || tail -5 gpurun_out/c2/build_dual.log
for name in one dual one2 dual2; do
  l=paper_conf_asplos_lis0l0c17_b200/libctaclust.so; case $name in dual*) l=$lib;; esac
  CTACLUST_LIB=$PWD/$l timeout 900 python bench_suite.py gpurun_out/c2/suite_$name.json --only conv \
     --variants 'agent-row$|identity$|agent-tile8x8$|direct|static-row-m7|tbcluster-2' > gpurun_out/c2/suite_$name.log 2>&1
  echo "== $name rc=$?"; sed -i '/Warn\|Acsr/d' gpurun_out/c2/suite_$name.log
done
