make all > /dev/null 2>&1
timeout -k 10 900 python scripts/exp_r10.py spmv_persist gpurun_out/spmv_persist.json 2>&1 | cut -c1-400
for v in "def:--backend default" "agent:--backend agent --order row"; do n=${v%%:*}; args=${v#*:}
  for p in "" "--persist-x"; do
    timeout -k 5 300 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum --clock-control none -k 'regex:k_(agent|default)' -s 1 -c 1 --csv python scripts/ncu_target.py --kernel spmv $args --hot 16384 $p --warm 1 --reps 1 2>/dev/null | grep -E "dram__bytes_read|gpu__time" | awk -F'","' -v n="$n$p" '{print n, $(NF-2), $NF}'
  done
done
