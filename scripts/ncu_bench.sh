# launch list of the bench command (our kernels only) + one full capture of the
# dominant kernel (1 GPU).  usage: bash scripts/ncu_bench.sh TAG
TAG=${1:-r02}
OUT=gpurun_out/ncu_$TAG
mkdir -p $OUT
timeout -k 5 900 ncu --metrics gpu__time_duration.sum --clock-control none -k 'regex:k_(agent|default|redirect|static|strip)' -c 400 --csv \
   --log-file $OUT/bench_launches.csv python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-parity --no-ncu > $OUT/bench_under_ncu.log 2>&1
echo launches rc=$?
timeout -k 5 900 ncu --set full --import-source on --clock-control none -k 'regex:k_agent' -s 2 -c 2 \
   -o $OUT/full_atax_agent python scripts/ncu_target.py --kernel atax --backend agent --order col --warm 1 --reps 1 > $OUT/full_atax.log 2>&1
echo full_atax rc=$?
timeout -k 5 900 ncu --set full --import-source on --clock-control none -k 'regex:k_agent' -s 1 -c 1 \
   -o $OUT/full_bicg_agent python scripts/ncu_target.py --kernel bicg --backend agent --order col --warm 1 --reps 1 > $OUT/full_bicg.log 2>&1
echo full_bicg rc=$?
timeout -k 5 900 ncu --set full --import-source on --clock-control none -k 'regex:k_agent' -s 1 -c 1 \
   -o $OUT/full_jacobi_agent python scripts/ncu_target.py --kernel jacobi --backend agent --order row --warm 1 --reps 1 > $OUT/full_jac.log 2>&1
echo full_jacobi rc=$?
timeout -k 5 900 ncu --set full --import-source on --clock-control none -k 'regex:k_strip' -s 1 -c 1 \
   -o $OUT/full_jwave_agent python scripts/ncu_target.py --kernel jwave --backend agent --order col --fuse 8 --warm 1 --reps 1 > $OUT/full_jwave.log 2>&1
echo full_jwave rc=$?
# summaries on the box (the reports would exceed what gpurun copies back)
python scripts/ncu_full_summary.py $TAG > $OUT/summary.log 2>&1
cp profiles/$TAG/ncu_full_summary.md $OUT/ 2>/dev/null
for f in $OUT/*.ncu-rep; do ncu -i $f --page raw --csv > ${f%.ncu-rep}.raw.csv 2>/dev/null; done
rm -f $OUT/*.ncu-rep
