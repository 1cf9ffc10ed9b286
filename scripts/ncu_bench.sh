# launch list of the bench command + one full capture of the dominant kernel (1 GPU)
TAG=${1:-r01}
OUT=gpurun_out/ncu_$TAG
mkdir -p $OUT
timeout -k 5 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
   --log-file $OUT/bench_launches.csv python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > $OUT/bench_under_ncu.log 2>&1
echo launches rc=$?
timeout -k 5 900 ncu --set full --import-source on --clock-control none -k "regex:k_agent" -s 4 -c 2 \
   -o $OUT/full_bicg_agent python scripts/ncu_target.py --kernel bicg --backend agent --order col --warm 2 --reps 2 > $OUT/full.log 2>&1
echo full rc=$?
timeout -k 5 900 ncu --set full --import-source on --clock-control none -k "regex:k_default" -s 1 -c 1 \
   -o $OUT/full_bicg_default python scripts/ncu_target.py --kernel bicg --backend default --warm 1 --reps 1 > $OUT/full_def.log 2>&1
echo full_def rc=$?
