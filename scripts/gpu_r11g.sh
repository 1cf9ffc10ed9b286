for N in 2048 8192 16384; do for c in jacf jac; do for st in 3 4; do timeout -k 5 60 python scripts/probe_stages.py $c $st $N 2>&1 | tail -1; echo "$c $st $N rc=$?"; done; done; done
