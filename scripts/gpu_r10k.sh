mkdir -p gpurun_out/r10k
make all > gpurun_out/r10k/build.log 2>&1 || tail -20 gpurun_out/r10k/build.log
timeout -k 10 600 python -m pytest tests/test_gpu_kernels.py -q -x --timeout 400 -k "tbc" > gpurun_out/r10k/t_conv.log 2>&1; echo tconv=$?
timeout -k 10 600 python scripts/exp_r10.py tbc gpurun_out/r10k/tbc.json > gpurun_out/r10k/tbc.log 2>&1; echo tbc=$?
bash scripts/ncu_full.sh r10k conv3_tbc1:"--kernel conv3 --backend tbcluster --cluster 1" conv3_tbc2:"--kernel conv3 --backend tbcluster --cluster 2" > gpurun_out/r10k/ncu.log 2>&1
timeout -k 10 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sectors_srcunit_tex.sum --clock-control none -k 'regex:k_(conv_tbc|agent|default)' --csv --log-file gpurun_out/r10k/seq.csv python scripts/ncu_target.py --kernel conv3 --backend tbcluster --cluster 1 --warm 0 --reps 4 > /dev/null 2>&1
tail -2 gpurun_out/r10k/t_conv.log; cat gpurun_out/r10k/tbc.log | cut -c1-900
