# conv 7x7 merged staging (CC_CONV7_MERGE=2, one tile-code instance) vs unmerged, same box
mkdir -p gpurun_out/m7 build
make -s all > gpurun_out/m7/build.log 2>&1 || tail -20 gpurun_out/m7/build.log
lib=build/libctaclust_m2.so
make -s LIB=$lib PTXLOG=gpurun_out/m7/ptx_m2.log CC_DEFS="-DCC_CONV7_MERGE=2" $lib > gpurun_out/m7/build_m2.log 2>&1 || tail -5 gpurun_out/m7/build_m2.log
CTACLUST_LIB=$PWD/$lib timeout 600 python -m pytest tests/test_gpu_kernels.py -q -x -k "conv or stencil" --timeout 300 > gpurun_out/m7/t_m2.log 2>&1; echo t_m2=$?; tail -1 gpurun_out/m7/t_m2.log
for name in m1 m2 m1b m2b; do
  l=paper_conf_asplos_lis0l0c17_b200/libctaclust.so; case $name in m2*) l=$lib;; esac
  CTACLUST_LIB=$PWD/$l timeout 900 python bench_suite.py gpurun_out/m7/suite_$name.json --only conv \
     --variants 'agent-row$|identity$|agent-tile8x8$|agent-tile8x8-s|static-row-m7|agent-row-l2last' > gpurun_out/m7/suite_$name.log 2>&1
  echo "== $name rc=$?"; sed -i '/Warn\|Acsr/d' gpurun_out/m7/suite_$name.log
done
M=dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex.sum,gpu__time_duration.sum
for name in m1 m2; do
  l=paper_conf_asplos_lis0l0c17_b200/libctaclust.so; [ $name = m2 ] && l=$lib
  CTACLUST_LIB=$PWD/$l timeout -k 5 300 ncu --metrics $M --clock-control none -k 'regex:k_agent' -s 1 -c 1 --csv --log-file gpurun_out/m7/ncu_$name.csv python scripts/ncu_target.py --warm 1 --reps 1 --kernel conv7 --backend agent --order row > gpurun_out/m7/ncu_$name.log 2>&1
done
