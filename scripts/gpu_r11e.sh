mkdir -p gpurun_out/r11e
make all > gpurun_out/r11e/build.log 2>&1 || tail -20 gpurun_out/r11e/build.log
for st in 2 3 4; do timeout -k 10 600 python bench.py --config jacobi --fuse 3 --stages $st --no-cpu-baseline --no-e2e --no-parity > gpurun_out/r11e/bench_jacobi_f3s$st.log 2>&1; echo s$st=$?; done
timeout -k 10 600 python bench.py --config jacobi --fuse 3 --stages 3 --batch 8 --no-cpu-baseline --no-e2e --no-parity > gpurun_out/r11e/bench_jacobi_f3s3b8.log 2>&1
for f in gpurun_out/r11e/bench_jacobi*.log; do echo $f; grep '^{' $f | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['ms_per_step'], d['speedup_vs_default'], d['speedup_vs_identity'], d['roofline']['frac'])"; done
