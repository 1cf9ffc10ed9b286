# SpMV A/B over build-time knobs: parity, suite timing and ncu L1-hit / L2-sector
# readout per build.  Run under gpurun from the repo root.
#   VARIANTS="name:defs name:defs"   (defs: comma-separated -D list)
mkdir -p gpurun_out
M=lts__t_sectors_srcunit_tex.sum,lts__t_sectors_srcunit_tex_op_read.sum,l1tex__t_sector_hit_rate.pct,dram__bytes_read.sum,sm__warps_active.avg.pct_of_peak_sustained_active,gpu__time_duration.sum,smsp__inst_executed.sum
K='regex:k_(agent|default|redirect)'
for spec in ${VARIANTS:-base:}; do
  tag=${spec%%:*}; defs=$(echo ${spec#*:} | tr ',' ' ')
  touch paper_conf_asplos_lis0l0c17_b200/csrc/ctaclust.cu
  make all CC_DEFS="$defs" > gpurun_out/build_$tag.log 2>&1 || { tail gpurun_out/build_$tag.log; continue; }
  timeout -k 10 600 python -m pytest tests/test_gpu_kernels.py -q -k spmv --timeout 300 > gpurun_out/t_spmv_$tag.log 2>&1; echo "$tag tests=$?"
  tail -1 gpurun_out/t_spmv_$tag.log
  timeout -k 10 600 python bench_suite.py gpurun_out/suite_spmv_$tag.json --only spmv > gpurun_out/suite_spmv_$tag.log 2>&1; echo "$tag suite=$?"
  [ -n "$NO_NCU" ] && continue
  for v in "default:--backend default" "agent-row:--backend agent --order row"; do
    name=${v%%:*}; args=${v#*:}
    timeout -k 5 300 ncu --metrics $M --clock-control none -k "$K" -s 1 -c 1 --csv \
      --log-file gpurun_out/ncu_spmv_${tag}_$name.csv python scripts/ncu_target.py --warm 1 --reps 1 --kernel spmv $args \
      > gpurun_out/ncu_spmv_${tag}_$name.log 2>&1
    echo "ncu $tag $name rc=$?"
  done
done
