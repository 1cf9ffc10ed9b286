# Diagnostic: TB-cluster conv halo box height (CC_TBC_HALO) -- parity + suite rows
mkdir -p gpurun_out/tbc build
make -s all > gpurun_out/tbc/build.log 2>&1
for v in "base:" "h4:-DCC_TBC_HALO=4"; do
  name=${v%%:*}; defs=${v#*:}
  lib=paper_conf_asplos_lis0l0c17_b200/libctaclust.so
  if [ -n "$defs" ]; then
    lib=build/libctaclust_$name.so
    make -s LIB=$lib PTXLOG=gpurun_out/tbc/ptx_$name.log CC_DEFS="$defs" $lib > gpurun_out/tbc/build_$name.log 2>&1 || tail -5 gpurun_out/tbc/build_$name.log
    CTACLUST_LIB=$PWD/$lib timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k 'conv' --timeout 300 > gpurun_out/tbc/t_$name.log 2>&1; echo "t_$name=$?"; tail -1 gpurun_out/tbc/t_$name.log
  fi
  CTACLUST_LIB=$PWD/$lib timeout 900 python bench_suite.py gpurun_out/tbc/suite_$name.json --only conv --variants 'tbcluster|identity$|agent-row$' > gpurun_out/tbc/suite_$name.log 2>&1
  echo "== $name rc=$?"; sed -i '/Warn\|Acsr/d' gpurun_out/tbc/suite_$name.log
done
