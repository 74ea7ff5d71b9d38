"""Seeded synthetic checkpoint state shaped like the paper's workloads.

This module serves both sides (oracle tests and the CUDA path) and holds none of the
method's arithmetic: it only says which tensors exist (names, shapes, dtypes, in
registration order) and fills them with seeded bit patterns.

Shapes (after SURVEY.md §8(d)):
  c1  97 fp32 tensors, 64 MiB total, log-uniform sizes (BASELINE.json configs[0])
  c2  VGG-16 fp32 params + SGD momentum            (configs[1]; PAPER Table 3)
  c3  OPT-1.3B fp32 params + Adam m, v, step       (configs[2]; Table 3)
  c4  BLOOM-7b1 bf16 params + fp32 master, m, v, step (configs[3]; Table 3)
  c5  OPT-2.7B fp32 params + Adam m, v, step       (configs[4]; Table 3)
  bert BERT-large (QA head) fp32 + Adam            (north_star list; Table 3)
Model inventories are written out analytically in ``model.parameters()`` order; a
CPU test cross-checks them against torchvision / transformers on the meta device.
Registration order (R11): per parameter ``[param, (fp32 master), exp_avg | momentum,
exp_avg_sq, step]``.
"""
from __future__ import annotations

from dataclasses import dataclass
from math import prod

import numpy as np

# dtype codes recorded in the registration (and hashed into layout_crc)
DTYPE_CODE = {"u8": 0, "f32": 1, "bf16": 2, "f16": 3, "f64": 4, "i64": 5, "i32": 6}
DTYPE_SIZE = {"u8": 1, "f32": 4, "bf16": 2, "f16": 2, "f64": 8, "i64": 8, "i32": 4}


@dataclass(frozen=True)
class TensorSpec:
    name: str
    shape: tuple
    dtype: str = "f32"
    kind: str = "param"  # param | master | momentum | exp_avg | exp_avg_sq | step | synthetic | zeros | const | nan | denormal

    @property
    def numel(self) -> int:
        return int(prod(self.shape)) if self.shape else 1

    @property
    def nbytes(self) -> int:
        return self.numel * DTYPE_SIZE[self.dtype]

    @property
    def code(self) -> int:
        return DTYPE_CODE[self.dtype]


# ---------------------------------------------------------------- model inventories
def vgg16_params():
    cfg = [64, 64, "M", 128, 128, "M", 256, 256, 256, "M", 512, 512, 512, "M", 512, 512, 512, "M"]
    out, cin, idx = [], 3, 0
    for v in cfg:
        if v == "M":
            idx += 1
            continue
        out += [(f"features.{idx}.weight", (v, cin, 3, 3)), (f"features.{idx}.bias", (v,))]
        cin = v
        idx += 2  # conv + relu
    for i, (a, b) in zip((0, 3, 6), ((512 * 7 * 7, 4096), (4096, 4096), (4096, 1000))):
        out += [(f"classifier.{i}.weight", (b, a)), (f"classifier.{i}.bias", (b,))]
    return out


def opt_params(hidden, layers, ffn, vocab=50272, max_pos=2048):
    h = hidden
    out = [("model.decoder.embed_tokens.weight", (vocab, h)),
           ("model.decoder.embed_positions.weight", (max_pos + 2, h)),
           ("model.decoder.final_layer_norm.weight", (h,)), ("model.decoder.final_layer_norm.bias", (h,))]
    for l in range(layers):
        p = f"model.decoder.layers.{l}."
        for proj in ("k_proj", "v_proj", "q_proj", "out_proj"):
            out += [(p + f"self_attn.{proj}.weight", (h, h)), (p + f"self_attn.{proj}.bias", (h,))]
        out += [(p + "self_attn_layer_norm.weight", (h,)), (p + "self_attn_layer_norm.bias", (h,)),
                (p + "fc1.weight", (ffn, h)), (p + "fc1.bias", (ffn,)),
                (p + "fc2.weight", (h, ffn)), (p + "fc2.bias", (h,)),
                (p + "final_layer_norm.weight", (h,)), (p + "final_layer_norm.bias", (h,))]
    return out


def bloom_params(hidden=4096, layers=30, vocab=250880):
    h = hidden
    out = [("transformer.word_embeddings.weight", (vocab, h)),
           ("transformer.word_embeddings_layernorm.weight", (h,)),
           ("transformer.word_embeddings_layernorm.bias", (h,))]
    for l in range(layers):
        p = f"transformer.h.{l}."
        out += [(p + "input_layernorm.weight", (h,)), (p + "input_layernorm.bias", (h,)),
                (p + "self_attention.query_key_value.weight", (3 * h, h)),
                (p + "self_attention.query_key_value.bias", (3 * h,)),
                (p + "self_attention.dense.weight", (h, h)), (p + "self_attention.dense.bias", (h,)),
                (p + "post_attention_layernorm.weight", (h,)), (p + "post_attention_layernorm.bias", (h,)),
                (p + "mlp.dense_h_to_4h.weight", (4 * h, h)), (p + "mlp.dense_h_to_4h.bias", (4 * h,)),
                (p + "mlp.dense_4h_to_h.weight", (h, 4 * h)), (p + "mlp.dense_4h_to_h.bias", (h,))]
    out += [("transformer.ln_f.weight", (h,)), ("transformer.ln_f.bias", (h,))]
    return out


def bert_large_qa_params(vocab=30522, h=1024, layers=24, ffn=4096, max_pos=512, types=2):
    out = [("bert.embeddings.word_embeddings.weight", (vocab, h)),
           ("bert.embeddings.position_embeddings.weight", (max_pos, h)),
           ("bert.embeddings.token_type_embeddings.weight", (types, h)),
           ("bert.embeddings.LayerNorm.weight", (h,)), ("bert.embeddings.LayerNorm.bias", (h,))]
    for l in range(layers):
        p = f"bert.encoder.layer.{l}."
        for q in ("query", "key", "value"):
            out += [(p + f"attention.self.{q}.weight", (h, h)), (p + f"attention.self.{q}.bias", (h,))]
        out += [(p + "attention.output.dense.weight", (h, h)), (p + "attention.output.dense.bias", (h,)),
                (p + "attention.output.LayerNorm.weight", (h,)), (p + "attention.output.LayerNorm.bias", (h,)),
                (p + "intermediate.dense.weight", (ffn, h)), (p + "intermediate.dense.bias", (ffn,)),
                (p + "output.dense.weight", (h, ffn)), (p + "output.dense.bias", (h,)),
                (p + "output.LayerNorm.weight", (h,)), (p + "output.LayerNorm.bias", (h,))]
    out += [("qa_outputs.weight", (2, h)), ("qa_outputs.bias", (2,))]
    return out


def _optimizer_state(params, optimizer, param_dtype="f32"):
    specs = []
    for name, shape in params:
        specs.append(TensorSpec(name, shape, param_dtype, "param"))
        if param_dtype != "f32":
            specs.append(TensorSpec(name + ".master", shape, "f32", "master"))
        if optimizer == "sgd":
            specs.append(TensorSpec(name + ".momentum_buffer", shape, "f32", "momentum"))
        else:
            specs.append(TensorSpec(name + ".exp_avg", shape, "f32", "exp_avg"))
            specs.append(TensorSpec(name + ".exp_avg_sq", shape, "f32", "exp_avg_sq"))
            specs.append(TensorSpec(name + ".step", (), "f32", "step"))  # fused/capturable Adam keeps a 0-d fp32 step
    return specs


def c1_tensors():
    """97 fp32 tensors, exactly 64 MiB: 96 floor(exp(U(0, ln 2^20))) sizes (PCG64 seed 0) with the
    first six forced to 1, 3, 5, 7, 33, 1023 numels, the last taking the remainder."""
    rng = np.random.default_rng(0)
    n = np.floor(np.exp(rng.uniform(0.0, np.log(2.0 ** 20), 96))).astype(np.int64).tolist()
    n[:6] = [1, 3, 5, 7, 33, 1023]
    n.append((64 << 20) // 4 - sum(n))
    kinds = ["synthetic"] * 97
    kinds[6], kinds[7], kinds[8], kinds[9] = "zeros", "const", "nan", "denormal"
    return [TensorSpec(f"t{i}", (k,), "f32", kinds[i]) for i, k in enumerate(n)]


CONFIGS = {
    "c1": dict(desc="synthetic 64 MiB fp32 state in 97 mixed-size tensors", chunk=4 << 20, n_inflight=2),
    "c2": dict(desc="VGG-16 fp32 params + SGD momentum", chunk=64 << 20, n_inflight=2),
    "c3": dict(desc="OPT-1.3B fp32 params + Adam", chunk=64 << 20, n_inflight=4),
    "c4": dict(desc="BLOOM-7b1 bf16 params + fp32 master + Adam", chunk=64 << 20, n_inflight=2),
    "c5": dict(desc="OPT-2.7B fp32 params + Adam", chunk=64 << 20, n_inflight=2),
    "bert": dict(desc="BERT-large QA fp32 params + Adam", chunk=64 << 20, n_inflight=2),
}


def config_tensors(cfg: str):
    if cfg == "c1":
        return c1_tensors()
    if cfg == "c2":
        return _optimizer_state(vgg16_params(), "sgd")
    if cfg == "c3":
        return _optimizer_state(opt_params(2048, 24, 8192), "adam")
    if cfg == "c4":
        return _optimizer_state(bloom_params(), "adam", param_dtype="bf16")
    if cfg == "c5":
        return _optimizer_state(opt_params(2560, 32, 10240), "adam")
    if cfg == "bert":
        return _optimizer_state(bert_large_qa_params(), "adam")
    raise KeyError(cfg)


# --------------------------------------------------------------------- value fill
_TORCH_DTYPE = None


def torch_dtype(d):
    import torch
    return {"u8": torch.uint8, "f32": torch.float32, "bf16": torch.bfloat16, "f16": torch.float16,
            "f64": torch.float64, "i64": torch.int64, "i32": torch.int32}[d]


def _structured_bytes(kind, nbytes, it):
    if kind == "zeros":
        return np.zeros(nbytes, dtype=np.uint8)
    words = -(-nbytes // 4)
    if kind == "const":
        w = np.full(words, 0x3F800000 + it, dtype=np.uint32)
    elif kind == "nan":  # quiet / signalling NaN payloads and -NaN
        w = np.resize(np.array([0x7FC00001, 0x7F800001, 0xFFBFFFFF, 0x7FFFFFFF], dtype=np.uint32), words) ^ np.uint32(it & 0xFF) << np.uint32(8)
    elif kind == "denormal":
        w = (np.arange(words, dtype=np.uint32) * np.uint32(2654435761) + np.uint32(it)) & np.uint32(0x807FFFFF)
    elif kind == "step":
        w = np.full(words, np.float32(it).view(np.uint32), dtype=np.uint32)
    else:
        raise KeyError(kind)
    return w.view(np.uint8)[:nbytes]


def make_state(specs, device, seed=0, it=0):
    """Allocates one torch tensor per spec on `device` and fills it with seeded bits.

    Random tensors draw uniform bytes from a torch Generator seeded by (seed, it, index);
    structured kinds (zeros / const / NaN payload / denormal / step) get fixed patterns
    that any float canonicalisation on the path would break.
    """
    import torch
    out = []
    for i, s in enumerate(specs):
        t = torch.empty(s.shape, dtype=torch_dtype(s.dtype), device=device)
        fill_tensor(t, s, seed, it, i)
        out.append(t)
    return out


def fill_tensor(t, s, seed, it, i):
    import torch
    flat = t.reshape(-1).view(torch.uint8) if t.dim() else t.reshape(1).view(torch.uint8)
    if s.nbytes == 0:
        return
    if s.kind in ("zeros", "const", "nan", "denormal", "step"):
        flat.copy_(torch.from_numpy(_structured_bytes(s.kind, s.nbytes, it)))
    else:
        g = torch.Generator(device=t.device)
        g.manual_seed((seed * 1_000_003 + it * 7919 + i) & 0x7FFFFFFFFFFFFFFF)
        flat.copy_(torch.randint(0, 256, (s.nbytes,), dtype=torch.uint8, generator=g, device=t.device))


def perturb_state(tensors, specs, seed, it):
    """Re-fills the state for iteration `it` (stands in for the optimizer update U)."""
    for i, (t, s) in enumerate(zip(tensors, specs)):
        fill_tensor(t, s, seed, it, i)


def host_bytes(t):
    """Raw bytes of a (device or host) tensor as a numpy uint8 array (host copy by torch)."""
    import torch
    flat = t.reshape(-1).view(torch.uint8) if t.dim() else t.reshape(1).view(torch.uint8)
    return flat.cpu().numpy()
