timeout -k 5 60 python scripts/probe_stages.py jac 3 8192 > gpurun_out/probe_jac3.log 2>&1; echo rc=$?
tail -20 gpurun_out/probe_jac3.log
CUDA_LAUNCH_BLOCKING=1 timeout -k 5 60 compute-sanitizer --print-limit 5 python scripts/probe_stages.py jac 3 2560 > gpurun_out/probe_jac3_san.log 2>&1; echo rc=$?
grep -E "Invalid|ERROR|at 0x|by thread" gpurun_out/probe_jac3_san.log | head -20
