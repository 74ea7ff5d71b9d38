for v in paper_conf_asplos_strati0k25_b200 build/va_old; do
echo "== $v"
PCC_LIB=$v/libpccheck.so ncu --metrics gpu__time_duration.sum --clock-control none --csv python tools/k1_bench.py --config c2 --cb 16777216 --reps 3 --unpack 2>/dev/null | grep -E "k_snapshot|k_finalize" | awk -F'","' '{print $5, $(NF)}' | tail -4
done
PCC_LIB=paper_conf_asplos_strati0k25_b200/libpccheck.so timeout 600 python bench.py --no-slowdown --no-cpu-baseline --steps 10 | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('restore', d['restore'], 'fin', d['finalize_ms'], 'k1', d['roofline']['launch_ms'])"
PCC_LIB=build/va_old/libpccheck.so timeout 600 python bench.py --no-slowdown --no-cpu-baseline --steps 10 | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('old restore', d['restore'], 'fin', d['finalize_ms'], 'k1', d['roofline']['launch_ms'])"
