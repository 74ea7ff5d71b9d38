"""The C-ABI library loads without a GPU and exports every symbol include/*.h declares."""
import ctypes
import glob
import os
import re

from conftest import ROOT


def _declared():
    names = set()
    for h in glob.glob(os.path.join(ROOT, "include", "*.h")):
        src = open(h).read()
        names |= set(re.findall(r"^PCC_API\s+[\w\s\*]+?\b(pcc_\w+)\s*\(", src, flags=re.M))
    return names


def test_headers_declare_the_boundary():
    d = _declared()
    for must in ["pcc_open", "pcc_register", "pcc_checkpoint", "pcc_guard", "pcc_poll", "pcc_wait", "pcc_commit",
                 "pcc_restore", "pcc_latest", "pcc_close", "pcc_k_pack", "pcc_k_unpack", "pcc_host_begin"]:
        assert must in d


def test_library_exports_every_declared_symbol():
    import paper_conf_asplos_strati0k25_b200 as pcc
    lib = ctypes.CDLL(pcc.LIB_PATH)
    missing = [n for n in sorted(_declared()) if not hasattr(lib, n)]
    assert not missing, missing
    # the Python binding marshals every declared call (and nothing undeclared)
    assert set(pcc.exported_symbols()) == _declared()


def test_struct_mirrors_match_the_build():
    """The ctypes mirrors of pcc_config / pcc_tensor / pcc_ckpt_info have the C sizes (a field
    added to the header without the binding, or the reverse, fails here)."""
    import paper_conf_asplos_strati0k25_b200 as pcc
    assert pcc._lib.pcc_struct_size(0) == ctypes.sizeof(pcc.Config)
    assert pcc._lib.pcc_struct_size(1) == ctypes.sizeof(pcc.Tensor)
    assert pcc._lib.pcc_struct_size(2) == ctypes.sizeof(pcc.Info)
    assert pcc._lib.pcc_struct_size(3) == ctypes.sizeof(pcc.RestoreInfo)
    assert pcc._lib.pcc_struct_size(7) == 0


def test_no_gpu_calls_fail_cleanly():
    import paper_conf_asplos_strati0k25_b200 as pcc
    assert pcc._lib.pcc_strerror(-pcc.ECORRUPT) == b"checksum mismatch"
    assert pcc.latest("/nonexistent/file") is None


def test_k_layout_matches_oracle():
    """Host-side layout of the product (no GPU) against the oracle's O1 on C1 and C2."""
    import oracle
    import paper_conf_asplos_strati0k25_b200 as pcc
    from synth import config_tensors
    for cfg, cb in (("c1", 4 << 20), ("c2", 64 << 20)):
        specs = config_tensors(cfg)
        fake = [(0x10000 * (i + 1), s.nbytes, s.code) for i, s in enumerate(specs)]
        off, end, c = pcc.k_layout(fake, 256, cb)
        o_off, o_end, o_c = oracle.layout([s.nbytes for s in specs], 256, cb)
        assert off == [int(x) for x in o_off] and end == o_end and c == o_c
