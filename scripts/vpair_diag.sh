mkdir -p gpurun_out/vp build
make -s all > gpurun_out/vp/build.log 2>&1
lib=build/libctaclust_inc.so
make -s LIB=$lib PTXLOG=gpurun_out/vp/ptx_inc.log CC_DEFS="-DCC_INC_DECODE=1" $lib > gpurun_out/vp/build_inc.log 2>&1
echo "-- default build"; timeout 600 python scripts/vpair_probe.py 2>&1 | grep -v Warn
echo "-- CC_INC_DECODE=1"; CTACLUST_LIB=$PWD/$lib timeout 600 python scripts/vpair_probe.py 2>&1 | grep -v Warn
