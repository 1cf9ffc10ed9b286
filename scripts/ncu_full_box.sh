# ncu_full.sh + summary on the box; keeps only the summary and the smallest report under gpurun_out
# usage: bash scripts/ncu_full_box.sh TAG name:args ...
TAG=$1
bash scripts/ncu_full.sh "$@"
python scripts/ncu_full_summary.py $TAG > gpurun_out/ncu_$TAG/summary.log 2>&1
cp profiles/$TAG/ncu_full_summary.md gpurun_out/ncu_$TAG/ 2>/dev/null
for f in gpurun_out/ncu_$TAG/*.ncu-rep; do ncu -i $f --page raw --csv > ${f%.ncu-rep}.raw.csv 2>/dev/null; done
rm -f gpurun_out/ncu_$TAG/*.ncu-rep
