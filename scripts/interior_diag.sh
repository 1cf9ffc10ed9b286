# conv: unmasked float4 stores for interior output blocks (CC_CONV_INTERIOR_FAST=1, default) vs masked stores
mkdir -p gpurun_out/if build
make -s all > gpurun_out/if/build.log 2>&1 || tail -20 gpurun_out/if/build.log
lib=build/libctaclust_nofast.so
make -s LIB=$lib PTXLOG=gpurun_out/if/ptx_nofast.log CC_DEFS="-DCC_CONV_INTERIOR_FAST=0" $lib > gpurun_out/if/build_nofast.log 2>&1
timeout -k 10 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "conv or stencil" --timeout 300 > gpurun_out/if/t.log 2>&1; echo t=$?; tail -1 gpurun_out/if/t.log
for name in fast nofast fast2 nofast2; do
  l=paper_conf_asplos_lis0l0c17_b200/libctaclust.so; case $name in nofast*) l=$lib;; esac
  CTACLUST_LIB=$PWD/$l timeout 600 python bench_suite.py gpurun_out/if/suite_$name.json --only conv --variants 'agent-row$|identity$|static-row-m7|tbcluster-2|l2last' > gpurun_out/if/suite_$name.log 2>&1
  echo "== $name rc=$?"; sed -i '/Warn\|Acsr/d' gpurun_out/if/suite_$name.log
done
