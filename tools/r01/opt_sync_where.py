"""Where does one OPT-1.3B training step synchronise?  (sync debug mode 'error' -> traceback)"""
import traceback

import torch
from transformers import OPTConfig, OPTForCausalLM

cfg = OPTConfig(hidden_size=2048, num_hidden_layers=24, ffn_dim=8192, num_attention_heads=32, vocab_size=50272,
                max_position_embeddings=2048, word_embed_proj_dim=2048)
net = OPTForCausalLM(cfg).cuda()
opt = torch.optim.Adam(net.parameters(), lr=1e-5, fused=True)
ids = torch.randint(0, cfg.vocab_size, (1, 2048), device="cuda")


def step():
    with torch.autocast("cuda", dtype=torch.bfloat16):
        loss = net(input_ids=ids, labels=ids).loss
    loss.backward()
    opt.step()
    opt.zero_grad(set_to_none=True)


for _ in range(2):
    step()
torch.cuda.synchronize()
torch.cuda.set_sync_debug_mode("error")
try:
    step()
    print("no sync")
except Exception:
    traceback.print_exc(limit=12)
