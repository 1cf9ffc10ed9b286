# Merged two-tile slots: stencil parity + suites (shipped build and a 4-agent 3x3 build).
mkdir -p gpurun_out build
make -s all > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_kernels.py tests/test_gpu_runtime.py tests/test_gpu_halo.py -q --timeout 600 > gpurun_out/t_merge.log 2>&1; echo "tests=$?"; tail -3 gpurun_out/t_merge.log
for v in "m5:" "m4:-DCC_CONV3_MIN_AGENTS=4"; do
  name=${v%%:*}; defs=${v#*:}
  lib=paper_conf_asplos_lis0l0c17_b200/libctaclust.so
  if [ -n "$defs" ]; then
    lib=build/libctaclust_$name.so
    make -s LIB=$lib PTXLOG=gpurun_out/ptx_$name.log CC_DEFS="$defs" $lib > gpurun_out/build_$name.log 2>&1 || tail -5 gpurun_out/build_$name.log
  fi
  CTACLUST_LIB=$PWD/$lib timeout 1200 python bench_suite.py gpurun_out/suite_mg_$name.json --only ${MERGE_SUITES:-jacobi,conv} --quick > gpurun_out/suite_mg_$name.log 2>&1
  echo "== $name rc=$?"
done
