# full ncu captures: conv 3x3 default / agent-row, Jacobi agent-row (one sweep)
mkdir -p gpurun_out/exp4
make all > gpurun_out/exp4/build.log 2>&1 || tail -20 gpurun_out/exp4/build.log
bash scripts/ncu_full.sh exp4 "conv3_default:--kernel conv3 --backend default" "conv3_agent:--kernel conv3 --backend agent --order row" \
   "jacobi_agent:--kernel jacobi --backend agent --order row" "conv3_identity:--kernel conv3 --backend identity"
