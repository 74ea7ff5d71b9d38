#!/usr/bin/env bash
# v7: the PCC_KCHECK build (bounds / alignment asserts, trap on violation) over the kernel + runtime
# parity suites; then the BLOOM-7B rank-0-of-8 proxy bench line (C4) with K1 v7
set -u
mkdir -p gpurun_out
o=gpurun_out/r02o.log; : > $o
PCC_LIB=build/kcheck/libpccheck.so timeout -s KILL 1500 python -m pytest tests/test_kernels_gpu.py tests/test_runtime_gpu.py tests/test_crash_gpu.py \
  -m gpu -q -p no:cacheprovider >> $o 2>&1; echo "kcheck rc=$?" >> $o
timeout -s KILL 3300 python bench.py --config c4 --emulate-world 8 > gpurun_out/r02o_bench_c4_rank0of8.json 2> gpurun_out/r02o_bench_c4.err; echo "c4 rc=$?" >> $o
cat $o | tail -8
