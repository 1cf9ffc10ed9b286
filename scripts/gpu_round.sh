# Full evidence pass for one round tag (1 GPU): correctness, bench line, suite,
# ncu L2-sector suite, bench launch list + full captures, categorizer.
#   bash scripts/gpu_round.sh r05
TAG=${1:-r07}
bash scripts/gpu_check.sh
bash scripts/ncu_suite.sh $TAG > gpurun_out/ncu_suite_$TAG.log 2>&1; echo "ncu_suite done"
bash scripts/ncu_bench.sh $TAG > gpurun_out/ncu_bench_$TAG.log 2>&1; echo "ncu_bench done"; cat gpurun_out/ncu_bench_$TAG.log
bash scripts/ncu_full.sh $TAG "matvec_static:--kernel matvec --backend static --order row --clusters 444" \
     "conv7_agent:--kernel conv7 --backend agent --order row" "conv3_agent:--kernel conv3 --backend agent --order row" "conv3_default:--kernel conv3 --backend default" > gpurun_out/ncu_full_$TAG.log 2>&1; cat gpurun_out/ncu_full_$TAG.log
timeout -k 10 1800 python scripts/categorize_run.py gpurun_out/categorize.json > gpurun_out/categorize.log 2>&1; echo "cat=$?"; tail -9 gpurun_out/categorize.log
timeout -k 10 300 python scripts/listing3.py gpurun_out/listing3.json > gpurun_out/listing3.log 2>&1; echo "listing3=$?"
