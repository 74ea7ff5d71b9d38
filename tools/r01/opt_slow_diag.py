"""OPT-1.3B slowdown diagnosis: host syncs in the training step, and the stall after a checkpoint
under different sinks / ring sizes / U-gate."""
import json
import os
import sys
import time
import warnings

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_asplos_strati0k25_b200 as pcc  # noqa: E402
from tools.slowdown import hf_slowdown  # noqa: E402

# 1) which ops of one OPT training step synchronise the host?
from transformers import OPTConfig, OPTForCausalLM  # noqa: E402
cfg = OPTConfig(hidden_size=2048, num_hidden_layers=24, ffn_dim=8192, num_attention_heads=32, vocab_size=50272,
                max_position_embeddings=2048, word_embed_proj_dim=2048)
net = OPTForCausalLM(cfg).cuda()
opt = torch.optim.Adam(net.parameters(), lr=1e-5, fused=True)
ids = torch.randint(0, cfg.vocab_size, (1, 2048), device="cuda")
for _ in range(2):
    with torch.autocast("cuda", dtype=torch.bfloat16):
        loss = net(input_ids=ids, labels=ids).loss
    loss.backward()
    opt.step()
    opt.zero_grad(set_to_none=True)
torch.cuda.synchronize()
torch.cuda.set_sync_debug_mode("warn")
with warnings.catch_warnings(record=True) as w:
    warnings.simplefilter("always")
    with torch.autocast("cuda", dtype=torch.bfloat16):
        loss = net(input_ids=ids, labels=ids).loss
    loss.backward()
    opt.step()
    opt.zero_grad(set_to_none=True)
torch.cuda.set_sync_debug_mode(0)
print("SYNC WARNINGS", len(w), [str(x.message)[:120] for x in w[:5]], flush=True)
del net, opt, ids, loss
torch.cuda.empty_cache()

for kw in [dict(flags=pcc.NULLSINK), dict(ring_bytes=2 * (16 << 30)), dict(use_guard=False), dict()]:
    r = hf_slowdown(pcc, "opt13", iters=30, **{k: v for k, v in kw.items()})
    print(json.dumps({"kw": {k: str(v) for k, v in kw.items()}, "slowdown_pct": round(r["slowdown_pct"], 2),
                      "host_max": r["host_ckpt_call_ms_max"], "its": [round(x) for x in r["iter_ms_ckpt_run"][8:13]],
                      "snap": r["contended"]["snapshot_ms"]}), flush=True)
