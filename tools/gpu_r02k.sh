#!/usr/bin/env bash
# the whole GPU suite on v7 (each file under its own timeout) + smoke + K2 launch times v7 vs v6
set -u
mkdir -p gpurun_out
o=gpurun_out/r02k_pytest.log; : > $o
for f in tests/test_kernels_gpu.py tests/test_runtime_gpu.py tests/test_crash_gpu.py tests/test_dp_gpu.py \
         tests/test_dp_crash_gpu.py tests/test_tuner.py tests/test_fullsize_gpu.py; do
  echo "== $f" >> $o
  timeout -s KILL 2000 python -m pytest $f -m gpu -q -p no:cacheprovider --durations=5 >> $o 2>&1
  echo "rc=$?" >> $o
done
timeout -s KILL 120 python -c "import __graft_entry__ as g; g.smoke()" >> $o 2>&1; echo "smoke rc=$?" >> $o
for impl in v7 v6; do
  for cfg in c2 c3; do
    PCC_KIMPL=$impl timeout -s KILL 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_snap" --csv \
      --log-file gpurun_out/r02k_k2_${impl}_${cfg}.csv python tools/k1_bench.py --config $cfg --reps 4 --unpack > /dev/null 2>&1
    echo "k2 $impl $cfg rc=$?" >> $o
  done
done
grep -E "^==|passed|failed|rc=|error|smoke ok" $o | tail -40
