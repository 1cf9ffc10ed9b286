mkdir -p gpurun_out/r11d
make all > gpurun_out/r11d/build.log 2>&1 || tail -20 gpurun_out/r11d/build.log
timeout -k 10 900 python -m pytest tests/test_gpu_sharded.py -q --timeout 600 -k "fused or jacobi" > gpurun_out/r11d/t.log 2>&1; echo t=$?
for f in 2 3 4; do timeout -k 10 600 python bench.py --config jacobi --fuse $f --no-cpu-baseline --no-e2e > gpurun_out/r11d/bench_jacobi_fuse$f.log 2>&1; echo bj$f=$?; done
tail -3 gpurun_out/r11d/t.log; grep -E "^FAILED" gpurun_out/r11d/t.log | head
for f in gpurun_out/r11d/bench_jacobi*.log; do echo $f; grep '^{' $f | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d.get('sweeps_per_second'), d['speedup_vs_default'], d['speedup_vs_identity'], d['roofline']['frac'], d['parity']['ok'])"; done
