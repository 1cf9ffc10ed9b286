# compute-sanitizer over tiny launches of every backend / body (scripts/sanitize_targets.py).
# usage (GPU box, repo root): bash scripts/sanitize.sh OUTDIR
OUT=${1:-gpurun_out/san}
mkdir -p $OUT
CS=/usr/local/cuda/bin/compute-sanitizer
for tool in memcheck racecheck synccheck initcheck; do
  for grp in ${SAN_GROUPS:-runtime gemv stencil tbc halo spmv wave}; do
    timeout -k 10 900 $CS --tool $tool --print-limit 20 --error-exitcode 9 \
      python scripts/sanitize_targets.py $grp > $OUT/${tool}_${grp}.log 2>&1
    rc=$?
    echo "$tool $grp rc=$rc $(grep -E 'ERROR SUMMARY|RACECHECK SUMMARY|SOME FAILED|ALL OK' $OUT/${tool}_${grp}.log | tr '\n' ' ')"
  done
done
