"""Where does the VGG-16 checkpoint-every-10 slowdown go?  Runs tools/slowdown.vgg16_slowdown
under several variants (K1 grid cap, sink, U-gate on/off) and prints one JSON line each:
slowdown %, the extra ms per iteration position, the host time of pcc_checkpoint."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))


def main():
    import paper_conf_asplos_strati0k25_b200 as pcc
    from tools.slowdown import vgg16_slowdown
    g = os.environ.get("DIAG_GRAPHS") == "1"
    variants = [
        dict(),
        dict(pack_ctas=74),
        dict(pack_ctas=32),
        dict(pack_ctas=16),
        dict(use_guard=False),
        dict(flags=pcc.NULLSINK),
        dict(chunk_bytes=16 << 20),
        dict(pack_ctas=8),
    ]
    pace = float(os.environ.get("PCC_D2H_GBS", "0"))
    quantum = int(float(os.environ.get("PCC_D2H_QUANTUM_MIB", "0")) * (1 << 20))
    for v in variants:
        v["graphs"] = g
        v["d2h_gbs"] = pace
        v["d2h_quantum"] = quantum
    only = os.environ.get("DIAG_ONLY")
    for i, v in enumerate(variants):
        if only and str(i) not in only.split(","):
            continue
        kw = dict(v)
        r = vgg16_slowdown(pcc, iters=60, every=10, runs=3, **kw)
        r["variant"] = {k: (hex(x) if k == "flags" else x) for k, x in v.items()}
        r["pack_prio"] = os.environ.get("PCC_PACK_PRIO", "high")
        r["pace"] = os.environ.get("PCC_D2H_GBS")
        r["extra_ms_by_pos"] = [round(x, 3) for x in r["extra_ms_by_pos"]]
        print(json.dumps(r), flush=True)


if __name__ == "__main__":
    main()
