"""The synthetic state generator: inventories and sizes (SURVEY §8 size table)."""
import pytest

import oracle
from synth import config_tensors, vgg16_params, opt_params, bloom_params, bert_large_qa_params, make_state

EXPECTED = {  # tensors, state bytes, chunk bytes, chunks  (SURVEY.md §8 "Config sizes", [verified] there)
    "c2": (64, 1_106_860_352, 64 << 20, 17),
    "c3": (1552, 15_789_098_512, 64 << 20, 236),
    "c4": (1825, 98_966_226_356, 64 << 20, 1475),
    "c5": (2064, 31_819_163_664, 64 << 20, 475),
}


@pytest.mark.parametrize("cfg", sorted(EXPECTED))
def test_config_sizes(cfg):
    specs = config_tensors(cfg)
    n, total, cb, chunks = EXPECTED[cfg]
    assert len(specs) == n
    assert sum(s.nbytes for s in specs) == total
    off, end, c = oracle.layout([s.nbytes for s in specs], 256, cb)
    assert c == chunks


def test_c2_4mib_chunks():
    specs = config_tensors("c2")
    assert oracle.layout([s.nbytes for s in specs], 256, 4 << 20)[2] == 264


def test_c1_edge_mix():
    specs = config_tensors("c1")
    nb = [s.nbytes for s in specs]
    assert sum(1 for n in nb if n < 16) == 10
    assert sum(1 for n in nb if n % 16) == 66
    assert max(nb) == 26_411_248


def test_inventories_match_model_libraries():
    torch = pytest.importorskip("torch")
    tv = pytest.importorskip("torchvision")
    tf = pytest.importorskip("transformers")
    with torch.device("meta"):
        ref = {
            "vgg": [(n, tuple(p.shape)) for n, p in tv.models.vgg16(weights=None).named_parameters()],
            "opt13": [(n, tuple(p.shape)) for n, p in tf.OPTForCausalLM(tf.OPTConfig(
                hidden_size=2048, num_hidden_layers=24, ffn_dim=8192, num_attention_heads=32, vocab_size=50272,
                max_position_embeddings=2048, word_embed_proj_dim=2048)).named_parameters()],
            "bloom": [(n, tuple(p.shape)) for n, p in tf.BloomForCausalLM(tf.BloomConfig(
                vocab_size=250880, hidden_size=4096, n_layer=30, n_head=32)).named_parameters()],
        }
    assert ref["vgg"] == vgg16_params()
    assert ref["opt13"] == opt_params(2048, 24, 8192)
    assert ref["bloom"] == bloom_params()


def test_make_state_deterministic_cpu():
    specs = config_tensors("c1")[:12]
    a = make_state(specs, "cpu", seed=3, it=5)
    b = make_state(specs, "cpu", seed=3, it=5)
    c = make_state(specs, "cpu", seed=3, it=6)
    import torch
    assert all(torch.equal(x.view(-1).view(torch.uint8), y.view(-1).view(torch.uint8)) for x, y in zip(a, b))
    assert any(not torch.equal(x.view(-1).view(torch.uint8), y.view(-1).view(torch.uint8))
               for x, y in zip(a, c) if x.numel() > 8)
