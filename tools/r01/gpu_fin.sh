set -u
timeout 900 python -m pytest tests/test_kernels_gpu.py tests/test_runtime_gpu.py -q -x -p no:cacheprovider 2>&1 | tail -2
python tools/k1_bench.py --config c2 --cb 16777216 --reps 8
python tools/k1_bench.py --config c3 --reps 4
