#!/usr/bin/env bash
# the whole GPU suite (each file under its own timeout) + the launch list of the bench's own kernels
set -u
mkdir -p gpurun_out
o=gpurun_out/r02f_pytest.log; : > $o
for f in tests/test_runtime_gpu.py tests/test_kernels_gpu.py tests/test_crash_gpu.py tests/test_dp_gpu.py \
         tests/test_dp_crash_gpu.py tests/test_tuner.py tests/test_fullsize_gpu.py; do
  echo "== $f" >> $o
  timeout -s KILL 2000 python -m pytest $f -m gpu -q -p no:cacheprovider --durations=5 >> $o 2>&1
  echo "rc=$?" >> $o
done
timeout -s KILL 120 python -c "import __graft_entry__ as g; g.smoke()" >> $o 2>&1; echo "smoke rc=$?" >> $o
timeout -s KILL 900 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_snapshot|k_fold|k_chunk" -c 300 --csv \
  --log-file gpurun_out/r02f_launches.csv python bench.py --steps 5 --warmup 3 --no-slowdown --no-cpu-baseline \
  > gpurun_out/r02f_bench_under_ncu.log 2>&1
echo "ncu rc=$?" >> $o
grep -E "^==|passed|failed|rc=|error|smoke ok" $o | tail -40
