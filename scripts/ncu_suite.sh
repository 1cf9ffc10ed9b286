# L2-sector / L1-hit / DRAM evidence for default vs clustered CTA order, every config.
# Run under gpurun from the repo root:  bash scripts/ncu_suite.sh [tag]
TAG=${1:-r02}
OUT=gpurun_out/ncu_$TAG
mkdir -p $OUT
M=lts__t_sectors.sum,lts__t_sectors_srcunit_tex.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_write.sum,lts__t_sectors_srcunit_tex_op_red.sum,lts__t_sectors_srcunit_tex_op_atom.sum,lts__t_sector_hit_rate.pct,l1tex__t_sector_hit_rate.pct,l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__warps_active.avg.pct_of_peak_sustained_active,gpu__time_duration.sum
K='regex:k_(agent|static|default|redirect|conv_tbc)'
run() {  # name, per-call launches, args...
  name=$1; per=$2; shift 2
  timeout -k 5 300 ncu --metrics $M --clock-control none -k "$K" -s $per -c $per --csv \
     --log-file $OUT/$name.csv python scripts/ncu_target.py --warm 1 --reps 1 "$@" > $OUT/$name.log 2>&1
  echo "$name rc=$?"
}
run matvec_default 1 --kernel matvec --backend default
run matvec_default-direct 1 --kernel matvec --backend default --staging direct
run matvec_agent-row 1 --kernel matvec --backend agent --order row
run matvec_agent-col 1 --kernel matvec --backend agent --order col
run matvec_agent-row-direct 1 --kernel matvec --backend agent --order row --staging direct
run matvec_identity 1 --kernel matvec --backend identity
run matvec_static-row-m2 1 --kernel matvec --backend static --order row --clusters 296
run matvec_static-row-m3 1 --kernel matvec --backend static --order row --clusters 444
for k in atax bicg mvt; do
  per=1; [ $k = atax ] && per=2
  run ${k}_default $per --kernel $k --backend default
  run ${k}_default-direct $per --kernel $k --backend default --staging direct
  run ${k}_agent-col $per --kernel $k --backend agent --order col
  run ${k}_agent-row $per --kernel $k --backend agent --order row
  run ${k}_agent-col-direct $per --kernel $k --backend agent --order col --staging direct
  run ${k}_identity $per --kernel $k --backend identity
  run ${k}_static-col-m3 $per --kernel $k --backend static --order col --clusters 444
done
run atax_fused_agent-row 1 --kernel atax_fused --backend agent --order row
run atax_fused_identity 1 --kernel atax_fused --backend identity
run atax_fused_static-row-m1 1 --kernel atax_fused --backend static --order row --clusters 148
for k in jacobi conv3 conv7; do
  run ${k}_default 1 --kernel $k --backend default
  run ${k}_default-l1 1 --kernel $k --backend default --staging l1
  run ${k}_default-direct 1 --kernel $k --backend default --staging direct
  run ${k}_agent-row 1 --kernel $k --backend agent --order row
  run ${k}_agent-tile8 1 --kernel $k --backend agent --order tile --tile 8x8
  run ${k}_agent-tile8-l1 1 --kernel $k --backend agent --order tile --tile 8x8 --staging l1
  run ${k}_agent-tile8-direct 1 --kernel $k --backend agent --order tile --tile 8x8 --staging direct
  run ${k}_agent-row-l1 1 --kernel $k --backend agent --order row --staging l1
  run ${k}_identity 1 --kernel $k --backend identity
  run ${k}_static-row-m4 1 --kernel $k --backend static --order row --clusters 592
done
for k in conv3 conv7; do
  run ${k}_tbc1 1 --kernel $k --backend tbcluster --cluster 1
  run ${k}_tbc2 1 --kernel $k --backend tbcluster --cluster 2
  run ${k}_tbc4 1 --kernel $k --backend tbcluster --cluster 4
  run ${k}_tbc8 1 --kernel $k --backend tbcluster --cluster 8
done
run conv7_static-row-m7 1 --kernel conv7 --backend static --order row --clusters 1036
run spmv_default 1 --kernel spmv --backend default
run spmv_agent-row 1 --kernel spmv --backend agent --order row
run spmv_identity 1 --kernel spmv --backend identity
run spmv_default-hot 1 --kernel spmv --backend default --hot 16384
run spmv_agent-row-hot 1 --kernel spmv --backend agent --order row --hot 16384
run hist_default 1 --kernel hist --backend default
run hist_agent-row 1 --kernel hist --backend agent --order row
run hist_identity 1 --kernel hist --backend identity
