# SpMV gather batch size sweep (diagnostic builds) + parity of the shipped build.
mkdir -p gpurun_out build
make -s all > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests/test_gpu_kernels.py -q -k "spmv" --timeout 600 > gpurun_out/t_spmv.log 2>&1; echo "spmv tests=$?"; tail -2 gpurun_out/t_spmv.log
for v in "gb8:" "gb4:-DCC_SPMV_GB=4" "gb16:-DCC_SPMV_GB=16" "gb16m4:-DCC_SPMV_GB=16 -DCC_SPMV_MIN_AGENTS=4"; do
  name=${v%%:*}; defs=${v#*:}
  lib=paper_conf_asplos_lis0l0c17_b200/libctaclust.so
  if [ -n "$defs" ]; then
    lib=build/libctaclust_$name.so
    make -s LIB=$lib PTXLOG=gpurun_out/ptx_$name.log CC_DEFS="$defs" $lib > gpurun_out/build_$name.log 2>&1 || tail -5 gpurun_out/build_$name.log
  fi
  CTACLUST_LIB=$PWD/$lib timeout 900 python bench_suite.py gpurun_out/suite_sp_$name.json --only spmv > gpurun_out/suite_sp_$name.log 2>&1
  echo "== $name rc=$?"
done
