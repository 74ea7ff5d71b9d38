#!/usr/bin/env bash
# K1 A/B on one box: the default build vs compile-time variants (tools/build_variant.sh builds
# them here; PCC_LIB selects one), two interleaved passes, C2 at the bench's 16 MiB chunks and C3.
set -u
mkdir -p gpurun_out
out=gpurun_out/k1_variants.jsonl
: > $out
for pass in 1 2; do
  for v in default $(ls -d build/v*/ 2>/dev/null | xargs -n1 basename); do
    lib=paper_conf_asplos_strati0k25_b200/libpccheck.so
    [ "$v" != default ] && lib=build/$v/libpccheck.so
    for c in "c2 --cb 16777216" "c3"; do
      r=$(PCC_LIB=$lib timeout 300 python tools/k1_bench.py --config $c --reps 8 2>&1 | tail -1)
      echo "{\"variant\": \"$v\", \"pass\": $pass, \"res\": $r}" >> $out
    done
  done
done
cat $out
