# round-2 evidence pass: GPU suite, sanitizer racecheck (runtime fix), bench every config, ncu suite + bench launch list
mkdir -p gpurun_out/r10i
make all > gpurun_out/r10i/build.log 2>&1 || tail -20 gpurun_out/r10i/build.log
timeout -k 10 1500 python -m pytest tests/ -m gpu -q --timeout 400 > gpurun_out/r10i/t_gpu.log 2>&1; echo gpu=$?
for g in runtime gemv stencil; do timeout -k 10 600 compute-sanitizer --tool racecheck --print-limit 20 --error-exitcode 9 python scripts/sanitize_targets.py $g > gpurun_out/r10i/racecheck_$g.log 2>&1; echo race_$g=$?; done
for c in atax jacobi conv3 conv7 spmv; do timeout -k 10 900 python bench.py --config $c > gpurun_out/r10i/bench_$c.log 2>&1; echo bench_$c=$?; done
bash scripts/ncu_suite.sh r10 > gpurun_out/r10i/ncu_suite.log 2>&1
bash scripts/ncu_bench.sh r10 > gpurun_out/r10i/ncu_bench.log 2>&1
tail -3 gpurun_out/r10i/t_gpu.log; cat gpurun_out/r10i/ncu_bench.log
