"""DESIGN §11 item 4: OPT-1.3B training slowdown vs the D2H pace (0 = the full link).
If the slowdown falls with the pace faster than the burst's duration grows, the burst's
rate (host DRAM / PCIe pressure on the launching thread) is the cause, not the copy count."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_strati0k25_b200 as pcc  # noqa: E402
from tools.slowdown import hf_slowdown  # noqa: E402

paces = [float(x) for x in (sys.argv[1:] or ["0", "45", "35", "25"])]
for g in paces:
    r = hf_slowdown(pcc, "opt13", d2h_gbs=g)
    keep = {k: r.get(k) for k in ("slowdown_pct", "iter_ms_no_ckpt", "iter_ms_ckpt", "d2h_gbs", "p99_ms")}
    keep["pace_gbs"] = g
    keep["iters_ms"] = [round(x, 1) for x in r.get("iter_ms_ckpt_run", [])[:20]]
    keep["contended_gbs"] = (r.get("contended") or {}).get("gbs")
    print(json.dumps(keep), flush=True)
