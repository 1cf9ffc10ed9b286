# wave Jacobi (R34): parity then timing
mkdir -p gpurun_out/jw
timeout -k 10 600 python -m pytest tests/test_gpu_jwave.py -q -x --timeout 300 > gpurun_out/jw/t.log 2>&1; echo t=$?
tail -5 gpurun_out/jw/t.log
timeout -k 10 600 python scripts/exp_jwave.py gpurun_out/jw/exp.json ${JW_FUSES:-2,3,4,5,6,8} > gpurun_out/jw/exp.log 2>&1; echo exp=$?
tail -50 gpurun_out/jw/exp.log
