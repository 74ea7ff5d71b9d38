#!/usr/bin/env bash
# compute-sanitizer memcheck / racecheck / synccheck over the K1/K2/finalize parity tests (small inputs)
set -u
mkdir -p gpurun_out
for t in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $t --print-limit 20 python -m pytest tests/test_kernels_gpu.py -q -x -p no:cacheprovider \
    -k "rfc or misaligned or partial or host_mapped or roundtrip" > gpurun_out/sanitizer_$t.txt 2>&1; echo "$t rc=$?"
  tail -3 gpurun_out/sanitizer_$t.txt
done
