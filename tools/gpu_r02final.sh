#!/usr/bin/env bash
# final round-2 validation of the committed tree: the whole -m gpu suite as the driver runs it, smoke, the default C3 bench line
set -u
mkdir -p gpurun_out
o=gpurun_out/r02final.log; : > $o
timeout -s KILL 3000 python -m pytest tests/ -x -q -m gpu -p no:cacheprovider >> $o 2>&1; echo "pytest-gpu rc=$?" >> $o
timeout -s KILL 120 python -c "import __graft_entry__ as g; g.smoke()" >> $o 2>&1; echo "smoke rc=$?" >> $o
timeout -s KILL 1500 python bench.py > gpurun_out/r02final_bench_c3.json 2> gpurun_out/r02final_bench_c3.err; echo "bench c3 rc=$?" >> $o
tail -6 $o
