"""DESIGN §11 item 4: OPT-1.3B slowdown with the chunks D2H-copied into a reused pinned staging
pool and dropped (PCC_NULLSINK) instead of into the registered tmpfs file mapping."""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import paper_conf_asplos_strati0k25_b200 as pcc  # noqa: E402
from tools.slowdown import hf_slowdown  # noqa: E402

r = hf_slowdown(pcc, "opt13", flags=pcc.NULLSINK)
print(json.dumps({"sink": "nullsink", "slowdown_pct": r.get("slowdown_pct"), "iter_ms_no_ckpt": r.get("iter_ms_no_ckpt"),
                  "iter_ms_ckpt": r.get("iter_ms_ckpt"),
                  "iters_ms": [round(x, 1) for x in r.get("iter_ms_ckpt_run", [])[:20]],
                  "contended_gbs": (r.get("contended") or {}).get("gbs")}))
