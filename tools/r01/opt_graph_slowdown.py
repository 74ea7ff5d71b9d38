"""DESIGN §11 item 4 (b): OPT-1.3B training (fp32 params, bf16 autocast, batch 1 x 2048,
Adam fused + capturable) with the whole step — zero_grad, forward, backward, optimizer — captured
as ONE CUDA graph, checkpointed every 10 iterations (R11 registration, 64 MiB chunks, MAPFILE),
against the same graph loop without checkpoints.  The U-gate is taken before the replay that
follows a checkpoint (conservative: the whole step waits for K1, not only the optimizer)."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402
import paper_conf_asplos_strati0k25_b200 as pcc  # noqa: E402
from transformers import OPTConfig, OPTForCausalLM  # noqa: E402

def opt13_graph_slowdown(attn="sdpa", host_lead=2, iters=40, every=10, ring_slices=1):
    """Returns the result dict printed by the script (see the module docstring)."""
    dev = torch.device("cuda", 0)
    cfg = OPTConfig(hidden_size=2048, num_hidden_layers=24, ffn_dim=8192, num_attention_heads=32, vocab_size=50272,
                    max_position_embeddings=2048, word_embed_proj_dim=2048)
    cfg._attn_implementation = attn
    net = OPTForCausalLM(cfg).to(dev).train()
    ids = torch.randint(0, cfg.vocab_size, (1, 2048), device=dev)
    mask = torch.ones(1, 2048, dtype=torch.long, device=dev)
    opt = torch.optim.Adam(net.parameters(), lr=1e-5, fused=True, capturable=True)

    def step():
        opt.zero_grad(set_to_none=False)
        with torch.autocast("cuda", dtype=torch.bfloat16, cache_enabled=False):
            loss = net(input_ids=ids, attention_mask=mask, labels=ids).loss
        loss.backward()
        opt.step()

    side = torch.cuda.Stream()
    side.wait_stream(torch.cuda.current_stream())
    with torch.cuda.stream(side):
        for _ in range(3):
            step()
    torch.cuda.current_stream().wait_stream(side)
    g = torch.cuda.CUDAGraph()
    with torch.cuda.graph(g):
        step()
    stream = torch.cuda.current_stream()
    state, _ = pcc.state_tensors(opt)
    path = f"/dev/shm/pcc_optgraph_{os.getpid()}.pcc"
    ck = pcc.PCCheck(path, chunk_bytes=64 << 20, max_inflight=2, flags=pcc.MAPFILE, staging_bytes=8 * (64 << 20), device=0,
                     ring_bytes=0 if ring_slices == 1 else ring_slices * (-(-sum(t.numel() * t.element_size() for t in state) // (64 << 20))) * (64 << 20))
    ck.register(state)

    def loop(n, checkpoint, it0):
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(n + 1)]
        evs[0].record(stream)
        hs = []
        for i in range(1, n + 1):
            if checkpoint and i % every == 1 and i > 1:
                ck.guard(stream)
            if host_lead and i > host_lead:
                evs[i - host_lead].synchronize()
            g.replay()
            if checkpoint and i % every == 0:
                th = time.perf_counter()
                hs.append(ck.checkpoint(it0 + i, stream))
                host_ms.append(round((time.perf_counter() - th) * 1e3, 2))
            evs[i].record(stream)
        evs[-1].synchronize()
        for h in hs:
            ck.wait(h)
        return [evs[i - 1].elapsed_time(evs[i]) for i in range(1, n + 1)]

    host_ms = []
    loop(5, False, 0)
    loop(12, True, 100)
    base = loop(iters, False, 0)
    host_ms.clear()
    withck = loop(iters, True, 1000)
    ck.drain()
    ck.close()
    os.unlink(path)
    mb, mc = sum(base) / len(base), sum(withck) / len(withck)
    return ({"model": f"OPT-1.3B, whole step as one CUDA graph ({attn} attention)", "every": every,
                      "iter_ms_no_ckpt": mb, "iter_ms_ckpt": mc, "slowdown_pct": 100 * (mc / mb - 1),
                      "iters_ms_ckpt": [round(x, 1) for x in withck], "host_lead": host_lead, "ring_slices": ring_slices, "host_ckpt_call_ms": host_ms,
                      "state_bytes": sum(t.numel() * t.element_size() for t in state), "tensors": len(state)})


if __name__ == "__main__":
    print(json.dumps(opt13_graph_slowdown(sys.argv[1] if len(sys.argv) > 1 else "sdpa",
                                          int(sys.argv[2]) if len(sys.argv) > 2 else 2,
                                          ring_slices=int(sys.argv[3]) if len(sys.argv) > 3 else 1)))
