set -u
OUT=gpurun_out; mkdir -p $OUT
ISO_GRAPH=1 ISO_KINDS=none,d2h,d2d_sm,ckpt timeout 600 python tools/slowdown_iso.py >> $OUT/iso2.jsonl 2>&1
for p in 50 40 30 20; do
  PCC_D2H_GBS=$p ISO_KINDS=none,ckpt timeout 600 python tools/slowdown_iso.py 2>&1 | grep ckpt >> $OUT/iso2.jsonl
done
PCC_D2H_GBS=30 PCC_D2H_QUANTUM_MIB=2 ISO_KINDS=none,ckpt timeout 600 python tools/slowdown_iso.py 2>&1 | grep ckpt >> $OUT/iso2.jsonl
PCC_D2H_GBS=30 ISO_GRAPH=1 ISO_KINDS=none,ckpt timeout 600 python tools/slowdown_iso.py 2>&1 | grep ckpt >> $OUT/iso2.jsonl
cat $OUT/iso2.jsonl | cut -c1-250
