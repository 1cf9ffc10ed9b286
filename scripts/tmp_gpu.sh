make all > /dev/null 2>&1
timeout -k 10 900 python bench.py --steps 20 --warmup 5 > gpurun_out/live_atax.log 2>&1; echo rc=$?
timeout -k 10 900 python bench.py --config conv3 --no-cpu-baseline > gpurun_out/live_conv3.log 2>&1; echo rc=$?
for f in atax conv3; do grep '^{' gpurun_out/live_$f.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(json.dumps(d['l2_sector_reduction'])[:900]); print(d['roofline'].get('traffic'), d['roofline'].get('traffic_source'), d['ms_per_step'])"; done
tail -5 gpurun_out/live_atax.log | cut -c1-300
