set -u
timeout 900 python -m pytest tests/test_kernels_gpu.py tests/test_runtime_gpu.py -q -x -p no:cacheprovider 2>&1 | tail -2
AB_UNPACK=1 bash tools/gpu_ab.sh 2>&1 | grep -v Warn | sed 's/"finalize_ms.*k1_gbs_algorithmic"/ gbs/'
