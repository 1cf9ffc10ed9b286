# full suite only (tag dir as $1)
mkdir -p gpurun_out/$1
make all > gpurun_out/$1/build.log 2>&1 || tail -20 gpurun_out/$1/build.log
timeout -k 10 1500 python bench_suite.py gpurun_out/$1/suite.json $2 > gpurun_out/$1/suite.log 2>&1; echo s=$?
sed -i '/Warn\|Acsr/d' gpurun_out/$1/suite.log
