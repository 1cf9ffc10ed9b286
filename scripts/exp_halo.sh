# CC_L2_HINT_HALO_LAST: parity + stencil suite rows + ncu DRAM bytes
mkdir -p gpurun_out/halo2
make -s all > gpurun_out/halo2/build.log 2>&1 || tail -20 gpurun_out/halo2/build.log
timeout -k 10 900 python -m pytest tests/test_gpu_kernels.py -q -x -k "jacobi or conv" --timeout 300 > gpurun_out/halo2/t.log 2>&1; echo t=$?; tail -2 gpurun_out/halo2/t.log
timeout -k 10 900 python bench_suite.py gpurun_out/halo2/suite.json --only jacobi,conv --variants 'l2halo|l2last|identity$|agent-row$' > gpurun_out/halo2/suite.log 2>&1; echo s=$?
sed -i '/Warn\|Acsr/d' gpurun_out/halo2/suite.log
M=dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex.sum,gpu__time_duration.sum
for v in "conv3_row:--kernel conv3 --backend agent --order row" "conv3_halo2:--kernel conv3 --backend agent --order row --l2 halo_last" \
         "jac_row:--kernel jacobi --backend agent --order row" "jac_halo2:--kernel jacobi --backend agent --order row --l2 halo_last"; do
  name=${v%%:*}; args=${v#*:}
  timeout -k 5 300 ncu --metrics $M --clock-control none -k 'regex:k_agent' -s 1 -c 1 --csv --log-file gpurun_out/halo2/ncu_$name.csv python scripts/ncu_target.py --warm 1 --reps 1 $args > gpurun_out/halo2/ncu_$name.log 2>&1
  echo "$name rc=$?"
done
