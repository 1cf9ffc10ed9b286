# A/B builds: TB-cluster stages / tile width / fence scope; conv 7x7 tile shape (RB, groups, agents)
mkdir -p gpurun_out/r10g
L=paper_conf_asplos_lis0l0c17_b200
make all > gpurun_out/r10g/build.log 2>&1 || tail -20 gpurun_out/r10g/build.log
bld() { make LIB=$L/lib_$1.so CC_DEFS="$2" PTXLOG=/tmp/p_$1.log > /dev/null 2>&1 & }
bld spg3 "-DCC_TBC_SPG=3"; bld spg4 "-DCC_TBC_SPG=4"; bld tw1 "-DCC_TBC_TW3=1 -DCC_TBC_SPG=3"; bld cta3 "-DCC_TBC_CTA_SCOPE=1 -DCC_TBC_SPG=3"
bld c7a "-DCC_CONV7_RB=8 -DCC_CONV7_GROUPS=2 -DCC_CONV7_AGENTS=6"; bld c7b "-DCC_CONV7_RB=8 -DCC_CONV7_GROUPS=4 -DCC_CONV7_AGENTS=4"; bld c7c "-DCC_CONV7_RB=8 -DCC_CONV7_GROUPS=4 -DCC_CONV7_AGENTS=3"; bld c7d "-DCC_CONV7_RB=4 -DCC_CONV7_GROUPS=4 -DCC_CONV7_AGENTS=4"
wait
for v in spg3 spg4 tw1 cta3; do
  echo "== $v"; EXP_CONV3_ONLY=1 CTACLUST_LIB=$PWD/$L/lib_$v.so timeout -k 10 300 python scripts/exp_r10.py tbc gpurun_out/r10g/tbc_$v.json 2>&1 | cut -c1-700
done
for v in c7a c7b c7c c7d; do
  echo "== $v"; CTACLUST_LIB=$PWD/$L/lib_$v.so timeout -k 10 300 python scripts/exp_r10.py conv7 gpurun_out/r10g/c7_$v.json 2>&1 | cut -c1-900
done
echo "== base"; timeout -k 10 300 python scripts/exp_r10.py conv7 gpurun_out/r10g/c7_base.json 2>&1 | cut -c1-900
