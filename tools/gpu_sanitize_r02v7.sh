#!/usr/bin/env bash
# (v7 kernels) compute-sanitizer memcheck / synccheck over the round-2 runtime (packer thread, inline K1, warm-up
# launches, D2H_UPFRONT, failed-window path) and the K1/K2 parity tests
set -u
mkdir -p gpurun_out
for t in memcheck synccheck racecheck; do
  timeout 1500 compute-sanitizer --tool $t --print-limit 20 python -m pytest tests/test_kernels_gpu.py tests/test_runtime_gpu.py -q -p no:cacheprovider \
    -k "rfc or misaligned or partial or host_mapped or roundtrip or file_matches_oracle or n_in_flight or small_ring or failed_k1 or unpack_into or many_rows or padding_only" \
    > gpurun_out/r02n_v7_sanitizer_$t.txt 2>&1; echo "$t rc=$?"
  tail -4 gpurun_out/r02n_v7_sanitizer_$t.txt
done
