set -u
OUT=gpurun_out; mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -q -x -p no:cacheprovider > $OUT/pytest_nt6.log 2>&1; echo "pytest nt6 rc=$?"; tail -3 $OUT/pytest_nt6.log
PCC_LIB=build/va_nt5/libpccheck.so timeout 600 python -m pytest tests/test_kernels_gpu.py -q -x -p no:cacheprovider 2>&1 | tail -2
bash tools/gpu_ab.sh 2>&1 | grep -v Warn
