# r05 pass: correctness (runtime, kernels, fused halo), bench line, full suite,
# and a launch list of fused vs plain slab sweeps.
mkdir -p gpurun_out
make all > gpurun_out/build.log 2>&1 || tail -20 gpurun_out/build.log
timeout -k 10 300 python __graft_entry__.py > gpurun_out/smoke.log 2>&1; echo smoke=$?
timeout -k 10 600 python -m pytest tests/test_gpu_runtime.py tests/test_gpu_comm.py tests/test_gpu_halo.py -q --timeout 300 > gpurun_out/t_runtime.log 2>&1; echo rt=$?
timeout -k 10 1500 python -m pytest tests/test_gpu_kernels.py -q --timeout 400 > gpurun_out/t_kernels.log 2>&1; echo k=$?
for f in smoke t_runtime t_kernels; do echo "== $f"; tail -n 4 gpurun_out/$f.log; done
timeout -k 10 1500 python bench_suite.py gpurun_out/suite.json ${SUITE_ARGS} > gpurun_out/suite.log 2>&1; echo s=$?
timeout -k 10 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/slab_launches.csv python scripts/slab_ncu.py > gpurun_out/slab_ncu.log 2>&1; echo ncu=$?
