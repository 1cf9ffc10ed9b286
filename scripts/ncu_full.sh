# one `ncu --set full` capture per listed variant (1 GPU).  usage: bash scripts/ncu_full.sh TAG name:args...
TAG=$1; shift
OUT=gpurun_out/ncu_$TAG
mkdir -p $OUT
for spec in "$@"; do
  name=${spec%%:*}; args=${spec#*:}
  timeout -k 5 600 ncu --set full --import-source on --clock-control none -k 'regex:k_(agent|static|default|redirect|conv_tbc|jwave|strip)' -s 1 -c 1 \
     -o $OUT/full_$name python scripts/ncu_target.py --warm 1 --reps 1 $args > $OUT/full_$name.log 2>&1
  echo "full_$name rc=$?"
done
