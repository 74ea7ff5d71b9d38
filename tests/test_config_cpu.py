"""pcc_open validates its configuration before touching the GPU (runs on CPU)."""
import pytest

pcc = pytest.importorskip("paper_conf_asplos_strati0k25_b200")


@pytest.mark.parametrize("kw", [
    dict(chunk_bytes=0),
    dict(chunk_bytes=100),                                   # not a multiple of 16
    dict(chunk_bytes=(4 << 20) + 16, flags=pcc.MAPFILE),     # MAPFILE needs 4096-multiples
    dict(chunk_bytes=(4 << 20) + 16, flags=pcc.ODIRECT),
    dict(max_inflight=0),
    dict(flags=pcc.ZEROCOPY),                                # Variant A needs the file mapping
    dict(flags=pcc.NULLSINK | pcc.MAPFILE),
    dict(flags=pcc.D2H_UPFRONT),                             # upfront copies go straight into the mapping
    dict(flags=pcc.NULLSINK | pcc.D2H_UPFRONT),
    dict(rank=2, world=2),
    dict(world=0),
    dict(world=2),                                           # no NCCL id and no callbacks
    dict(align=8),
])
def test_invalid_configs_rejected(tmp_path, kw):
    args = dict(path=str(tmp_path / "x.pcc"), chunk_bytes=4 << 20, max_inflight=2, flags=pcc.MAPFILE)
    args.update(kw)
    with pytest.raises(pcc.PCCError) as ei:
        pcc.PCCheck(**args)
    assert ei.value.code == pcc.EINVAL


def test_callbacks_must_come_in_pairs(tmp_path):
    with pytest.raises(pcc.PCCError) as ei:
        pcc.PCCheck(str(tmp_path / "x.pcc"), world=2, allreduce=lambda v, m: v, allgather=None)
    assert ei.value.code == pcc.EINVAL
