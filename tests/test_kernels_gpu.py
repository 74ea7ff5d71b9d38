"""K1 / K2 parity against the CPU oracle, bit-exact (tolerance 0 bytes), through the C ABI.

The oracle sees the state through an independent host copy (torch .cpu()); both sides get
the same seeded inputs from synth/.  Sizes span several 32 KiB tiles and ragged tails; the
RFC pin needs no oracle at all.
"""
import os

import numpy as np
import pytest

import oracle
from conftest import ROOT
from synth import config_tensors, make_state, host_bytes

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def pcc():
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    import paper_conf_asplos_strati0k25_b200 as p
    return p


def _pack_gpu(pcc, tensors, align, cb, first=0, count=None, dst=None):
    off, end, c = pcc.k_layout(tensors, align, cb)
    if count is None:
        count = c - first
    if dst is None:
        dst = torch.full((max(1, count * cb),), 0xA5, dtype=torch.uint8, device="cuda")  # stale bytes must vanish
    crc = torch.zeros(max(1, count), dtype=torch.int32, device="cuda")
    dig = torch.zeros(1, dtype=torch.int32, device="cuda")
    pcc.k_pack(tensors, dst.data_ptr(), crc.data_ptr(), dig.data_ptr(), align, cb, first, count)
    torch.cuda.synchronize()
    return (dst[:count * cb].cpu().numpy(), crc[:count].cpu().numpy().view(np.uint32).tolist(),
            int(dig.cpu().numpy().view(np.uint32)[0]))


def test_rfc_pin_on_gpu(pcc):
    """P4: four RFC 3720 patterns, ALIGN 256, CB 32 -> the golden CRC table (no oracle involved)."""
    pats = [bytes(32), b"\xff" * 32, bytes(range(32)), bytes(range(31, -1, -1))]
    ts = [torch.tensor(list(p), dtype=torch.uint8, device="cuda") for p in pats]
    img, crcs, dig = _pack_gpu(pcc, ts, 256, 32)
    exp = []
    for line in open(os.path.join(ROOT, "tests", "golden", "rfc_pack_pin.txt")):
        if line.strip() and not line.startswith("#"):
            exp.append(int(line.split()[1], 16))
    assert crcs == exp
    assert dig == oracle.crc32c(img)


def _oracle_side(tensors, align, cb, first=0, count=None):
    hb = [host_bytes(t) for t in tensors]
    img = oracle.pack(hb, align=align, chunk_bytes=cb, first_chunk=first, count=count)
    return img, [int(x) for x in oracle.chunk_crcs(img, cb)], oracle.crc32c(img)


@pytest.mark.parametrize("cb", [4 << 20, 64 << 10, 48, 32768 + 16, 3 * 32768 - 16])
def test_c1_full_image_parity(pcc, cb):
    specs = config_tensors("c1")
    ts = make_state(specs, "cuda", seed=11, it=3)
    img, crcs, dig = _pack_gpu(pcc, ts, 256, cb)
    o_img, o_crcs, o_dig = _oracle_side(ts, 256, cb)
    assert img.nbytes == o_img.nbytes
    diff = np.flatnonzero(img != o_img)
    assert diff.size == 0, f"{diff.size} bytes differ, first at {diff[:8]}"
    assert crcs == o_crcs
    assert dig == o_dig


@pytest.mark.parametrize("align", [16, 256, 4096])
def test_misaligned_sources_all_16_offsets(pcc, align):
    """Source views at every byte alignment 0..15 with ragged lengths (storage_offset views)."""
    base = torch.randint(0, 256, (1 << 20,), dtype=torch.uint8, device="cuda")
    rng = np.random.default_rng(5)
    ts = []
    pos = 0
    for k in range(48):
        a = k % 16
        n = int(rng.integers(0, 70000))
        start = ((pos + 4095) // 4096) * 4096 + a
        ts.append(base[start:start + n])
        pos = start + n
    img, crcs, dig = _pack_gpu(pcc, ts, align, 64 << 10)
    o_img, o_crcs, o_dig = _oracle_side(ts, align, 64 << 10)
    assert np.array_equal(img, o_img) and crcs == o_crcs and dig == o_dig


def test_partial_chunk_range_and_zero_sized(pcc):
    specs = config_tensors("c1")[:30]
    ts = make_state(specs, "cuda", seed=2, it=0)
    ts.insert(5, torch.empty(0, dtype=torch.float32, device="cuda"))
    ts.insert(9, torch.zeros((), dtype=torch.float32, device="cuda") + 3.5)  # 0-d
    off, end, c = pcc.k_layout(ts, 256, 65536)
    for first, count in ((0, 1), (1, 3), (c - 2, 2), (c // 2, c - c // 2)):
        img, crcs, dig = _pack_gpu(pcc, ts, 256, 65536, first, count)
        o_img, o_crcs, o_dig = _oracle_side(ts, 256, 65536, first, count)
        assert np.array_equal(img, o_img) and crcs == o_crcs and dig == o_dig


def test_pack_into_host_mapped_pinned_memory(pcc):
    """Variant A's store path: K1 writes straight into pinned host memory over PCIe."""
    specs = config_tensors("c1")
    ts = make_state(specs, "cuda", seed=4, it=1)
    off, end, c = pcc.k_layout(ts, 256, 4 << 20)
    dst = torch.full((c * (4 << 20),), 0x5A, dtype=torch.uint8).pin_memory()
    crc = torch.zeros(c, dtype=torch.int32, device="cuda")
    dig = torch.zeros(1, dtype=torch.int32, device="cuda")
    pcc.k_pack(ts, dst.data_ptr(), crc.data_ptr(), dig.data_ptr(), 256, 4 << 20)
    torch.cuda.synchronize()
    o_img, o_crcs, o_dig = _oracle_side(ts, 256, 4 << 20)
    assert np.array_equal(dst.numpy(), o_img)
    assert crc.cpu().numpy().view(np.uint32).tolist() == o_crcs


def test_unpack_roundtrip_and_detection(pcc):
    specs = config_tensors("c1")
    ts = make_state(specs, "cuda", seed=8, it=2)
    cb = 1 << 20
    off, end, c = pcc.k_layout(ts, 256, cb)
    img = torch.empty(c * cb, dtype=torch.uint8, device="cuda")
    crc = torch.zeros(c, dtype=torch.int32, device="cuda")
    dig = torch.zeros(1, dtype=torch.int32, device="cuda")
    pcc.k_pack(ts, img.data_ptr(), crc.data_ptr(), dig.data_ptr(), 256, cb)
    outs = [torch.full_like(t, 0) if t.dtype != torch.float32 else torch.full_like(t, float("nan")) for t in ts]
    bad = torch.zeros(c, dtype=torch.int32, device="cuda")
    nbad = torch.zeros(1, dtype=torch.int32, device="cuda")
    dig2 = torch.zeros(1, dtype=torch.int32, device="cuda")
    pcc.k_unpack(outs, img.data_ptr(), crc.data_ptr(), bad.data_ptr(), nbad.data_ptr(), dig2.data_ptr(), 256, cb)
    torch.cuda.synchronize()
    assert int(nbad.item()) == 0 and int(dig2.item()) == int(dig.item())
    for a, b in zip(ts, outs):
        assert np.array_equal(host_bytes(a), host_bytes(b))
    # flip one bit in chunk 7 and a 32-bit burst in chunk 12 -> exactly those two chunks flagged
    img[7 * cb + 12345] ^= 0x20
    img[12 * cb + 100:12 * cb + 104] ^= 0xFF
    pcc.k_unpack(outs, img.data_ptr(), crc.data_ptr(), bad.data_ptr(), nbad.data_ptr(), dig2.data_ptr(), 256, cb)
    torch.cuda.synchronize()
    assert int(nbad.item()) == 2
    assert np.flatnonzero(bad.cpu().numpy()).tolist() == [7, 12]


def test_c2_vgg_full_size_parity(pcc):
    """BASELINE configs[1] at full size (1.107 GB, 64 MiB chunks): full image, CRC table, digest."""
    specs = config_tensors("c2")
    ts = make_state(specs, "cuda", seed=0, it=0)
    img, crcs, dig = _pack_gpu(pcc, ts, 256, 64 << 20)
    o_img, o_crcs, o_dig = _oracle_side(ts, 256, 64 << 20)
    assert np.array_equal(img, o_img)
    assert crcs == o_crcs and dig == o_dig


def test_nccl_transport_selftest(pcc):
    """The library's own NCCL path (nccl_shim.hpp: dlopen, ncclCommInitRank, int64 MIN / MAX
    allreduce, byte allgather) on a real GPU: one rank, since one GPU cannot host two."""
    vals = [30, -1, 2**40 + 5, 0, 7]
    mn, mx, ok = pcc.nccl_selftest(vals)
    assert mn == vals and mx == vals and ok


def _unpack_gpu(pcc, outs, img, crc, align, cb):
    c = crc.numel()
    bad = torch.zeros(c, dtype=torch.int32, device="cuda")
    nbad = torch.zeros(1, dtype=torch.int32, device="cuda")
    dig = torch.zeros(1, dtype=torch.int32, device="cuda")
    pcc.k_unpack(outs, img.data_ptr(), crc.data_ptr(), bad.data_ptr(), nbad.data_ptr(), dig.data_ptr(), align, cb)
    torch.cuda.synchronize()
    return int(nbad.item()), int(dig.cpu().numpy().view(np.uint32)[0])


@pytest.mark.parametrize("cb", [64 << 10, 32768 + 16, 3 * 32768 - 16, 48])
def test_unpack_into_misaligned_views_ragged_chunks(pcc, cb):
    """K2's scatter: destinations at every byte alignment 0..15 with ragged lengths, chunk sizes
    whose last 8 KiB tile is ragged; every byte outside the views must stay untouched."""
    rng = np.random.default_rng(21)
    src_base = torch.randint(0, 256, (1 << 20,), dtype=torch.uint8, device="cuda")
    dst_base = torch.full((1 << 20,), 0x3C, dtype=torch.uint8, device="cuda")
    srcs, dsts, pos, spans = [], [], 0, []
    for k in range(40):
        a = int(rng.integers(0, 16))
        n = int(rng.integers(0, 20000))
        start = ((pos + 4095) // 4096) * 4096 + a
        srcs.append(src_base[start:start + n])
        dsts.append(dst_base[start:start + n])
        spans.append((start, n))
        pos = start + n
    off, end, c = pcc.k_layout(srcs, 256, cb)
    img = torch.empty(max(1, c * cb), dtype=torch.uint8, device="cuda")
    crc = torch.zeros(max(1, c), dtype=torch.int32, device="cuda")
    dig = torch.zeros(1, dtype=torch.int32, device="cuda")
    pcc.k_pack(srcs, img.data_ptr(), crc.data_ptr(), dig.data_ptr(), 256, cb)
    o_img, o_crcs, o_dig = _oracle_side(srcs, 256, cb)
    assert np.array_equal(img[:c * cb].cpu().numpy(), o_img)
    nbad, dig2 = _unpack_gpu(pcc, dsts, img, crc[:c], 256, cb)
    assert nbad == 0 and dig2 == o_dig
    expect = np.full(1 << 20, 0x3C, dtype=np.uint8)
    sb = src_base.cpu().numpy()
    for start, n in spans:
        expect[start:start + n] = sb[start:start + n]
    got = dst_base.cpu().numpy()
    assert np.array_equal(got, expect), f"{np.count_nonzero(got != expect)} bytes differ"


def test_many_rows_per_tile_align16(pcc):
    """align 16 and tiny tensors: up to hundreds of segment rows inside one 8 KiB tile (the
    producer / storer loop over rows in groups of 32), tiles that are all padding, ragged rows."""
    rng = np.random.default_rng(9)
    sizes = [int(x) for x in rng.integers(0, 90, 3000)]
    sizes[100:140] = [0] * 40
    ts = [torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda") for n in sizes]
    ts.append(torch.empty(0, dtype=torch.uint8, device="cuda"))
    for cb in (64 << 10, 8192 + 16 * 7):
        img, crcs, dig = _pack_gpu(pcc, ts, 16, cb)
        o_img, o_crcs, o_dig = _oracle_side(ts, 16, cb)
        assert np.array_equal(img, o_img) and crcs == o_crcs and dig == o_dig
        outs = [torch.zeros_like(t) for t in ts]
        off, end, c = pcc.k_layout(ts, 16, cb)
        g_img = torch.from_numpy(o_img).cuda()
        g_crc = torch.tensor(np.array(o_crcs, dtype=np.uint32).view(np.int32), device="cuda")
        nbad, dig2 = _unpack_gpu(pcc, outs, g_img, g_crc, 16, cb)
        assert nbad == 0 and dig2 == o_dig
        assert all(np.array_equal(host_bytes(a), host_bytes(b)) for a, b in zip(ts, outs))


def test_padding_only_tiles(pcc):
    """A 4096-B alignment leaves whole 8 KiB tiles without any row (all zeros in the image)."""
    ts = [torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda") for n in (5, 70000, 1, 24577)]
    img, crcs, dig = _pack_gpu(pcc, ts, 65536, 1 << 20)
    o_img, o_crcs, o_dig = _oracle_side(ts, 65536, 1 << 20)
    assert np.array_equal(img, o_img) and crcs == o_crcs and dig == o_dig


def test_register_path_kernels_v6_parity():
    """PCC_KIMPL=v6 (the register-path K1/K2 kept for same-box A/B) in its own process: C1 full
    image + CRC table + digest vs the oracle, and a K2 round trip."""
    import subprocess
    import sys
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    code = (
        "import sys, numpy as np, torch; sys.path.insert(0, %r); sys.path.insert(0, %r)\n"
        "import oracle, paper_conf_asplos_strati0k25_b200 as pcc\n"
        "from synth import config_tensors, make_state, host_bytes\n"
        "ts = make_state(config_tensors('c1'), 'cuda', seed=3, it=1); cb = 32768 + 16\n"
        "off, end, c = pcc.k_layout(ts, 256, cb)\n"
        "img = torch.empty(c * cb, dtype=torch.uint8, device='cuda'); crc = torch.zeros(c, dtype=torch.int32, device='cuda')\n"
        "dig = torch.zeros(1, dtype=torch.int32, device='cuda')\n"
        "pcc.k_pack(ts, img.data_ptr(), crc.data_ptr(), dig.data_ptr(), 256, cb); torch.cuda.synchronize()\n"
        "hb = [host_bytes(t) for t in ts]; o = oracle.pack(hb, 256, cb)\n"
        "assert np.array_equal(img.cpu().numpy(), o)\n"
        "assert crc.cpu().numpy().view(np.uint32).tolist() == [int(x) for x in oracle.chunk_crcs(o, cb)]\n"
        "assert int(dig.cpu().numpy().view(np.uint32)[0]) == oracle.crc32c(o)\n"
        "outs = [torch.zeros_like(t) for t in ts]; bad = torch.zeros(c, dtype=torch.int32, device='cuda')\n"
        "aux = torch.zeros(2, dtype=torch.int32, device='cuda')\n"
        "pcc.k_unpack(outs, img.data_ptr(), crc.data_ptr(), bad.data_ptr(), aux.data_ptr(), aux[1:].data_ptr(), 256, cb)\n"
        "torch.cuda.synchronize(); assert int(aux[0].item()) == 0\n"
        "assert all(np.array_equal(host_bytes(a), b) for a, b in zip(outs, hb))\n"
        "print('v6 ok')\n") % (ROOT, os.path.join(ROOT, "tests"))
    env = dict(os.environ, PCC_KIMPL="v6")
    r = subprocess.run([sys.executable, "-c", code], env=env, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0 and "v6 ok" in r.stdout, r.stdout + r.stderr
