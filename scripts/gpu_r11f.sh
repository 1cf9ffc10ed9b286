for c in jac jacf conv; do for st in 2 3 4 5; do timeout -k 5 60 python scripts/probe_stages.py $c $st 2>&1 | tail -1; echo "$c $st rc=$?"; done; done
