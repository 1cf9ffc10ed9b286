# conv/jacobi L2-hint rows under graph timing + conv7 agent full capture
mkdir -p gpurun_out/exp6
make all > gpurun_out/exp6/build.log 2>&1 || tail -20 gpurun_out/exp6/build.log
timeout -k 10 900 python bench_suite.py gpurun_out/exp6/suite.json --only conv,jacobi --variants 'l2|identity$|agent-row$|agent-tile' > gpurun_out/exp6/suite.log 2>&1; echo s=$?
sed -i '/Warn\|Acsr/d' gpurun_out/exp6/suite.log
bash scripts/ncu_full.sh exp6 "conv7_agent:--kernel conv7 --backend agent --order row"
