"""Crash consistency with real process death (SURVEY §4 "Integration"): a child process
checkpoints iter 10, then is SIGKILLed by PCC_FAULT somewhere inside iter 20's checkpoint; the
file must still restore iter 10 bit-exactly — through the oracle and through a fresh library
context that resumes on the same file (a persistent checkpoint always exists)."""
import os
import subprocess
import sys

import numpy as np
import pytest

import oracle
from conftest import ROOT
from synth import config_tensors, make_state, host_bytes

pytestmark = [pytest.mark.gpu, pytest.mark.timeout(300)]
torch = pytest.importorskip("torch")
CB = 4 << 20

CHILD = r"""
import os, sys
import numpy as np
sys.path.insert(0, sys.argv[3])
import torch
import paper_conf_asplos_strati0k25_b200 as pcc
from synth import config_tensors, make_state, perturb_state, host_bytes
specs = config_tensors("c1")
ts = make_state(specs, "cuda", seed=41, it=0)
ck = pcc.PCCheck(sys.argv[1], chunk_bytes=4 << 20, max_inflight=2, flags=pcc.MAPFILE | pcc.FSYNC)
ck.register(ts)
perturb_state(ts, specs, 41, 10)
ck.wait(ck.checkpoint(10))
np.save(sys.argv[2], np.concatenate([host_bytes(t) for t in ts]))
perturb_state(ts, specs, 41, 20)
ck.wait(ck.checkpoint(20))
sys.exit(7)  # the fault did not fire
"""

# (point, occurrence that falls inside iter 20's checkpoint).  C1's 17 chunks of 4 MiB land
# in two coalesced copies per checkpoint, so the 3rd copy is iter 20's first.
FAULTS = [("chunk", 3), ("header", 2), ("pointer", 2), ("mid_pointer", 2)]


@pytest.mark.parametrize("point,n", FAULTS)
def test_sigkill_inside_checkpoint_keeps_previous(tmp_path, point, n):
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    d = "/dev/shm" if os.path.isdir("/dev/shm") else str(tmp_path)
    path = os.path.join(d, f"pcc_crash_{os.getpid()}_{point}.pcc")
    save = str(tmp_path / "s10.npy")
    env = dict(os.environ, PCC_FAULT=f"{point}:{n}")
    try:
        r = subprocess.run([sys.executable, "-c", CHILD, path, save, ROOT], env=env, timeout=240,
                           capture_output=True, text=True)
        assert r.returncode == -9, (r.returncode, r.stderr[-2000:])
        s10 = np.load(save)
        specs = config_tensors("c1")
        nbytes = [s.nbytes for s in specs]
        rc, it, bad, outs = oracle.restore([path], 3, nbytes, [s.code for s in specs], 256, CB)
        assert rc == 0 and it == 10
        assert np.array_equal(np.concatenate(outs), s10)
        # a fresh library context resumes on the same file and restores the same bytes
        import paper_conf_asplos_strati0k25_b200 as pcc
        ts = make_state(specs, "cuda", seed=99, it=0)
        with pcc.PCCheck(path, chunk_bytes=CB, max_inflight=2, flags=pcc.MAPFILE) as ck:
            ck.register(ts)
            it, bad = ck.restore()
            assert it == 10 and bad == []
            assert np.array_equal(np.concatenate([host_bytes(t) for t in ts]), s10)
            # ... and keeps checkpointing after the crash: the next commit supersedes iter 10
            h = ck.checkpoint(30)
            ck.wait(h)
            assert pcc.latest(path) == (30, 30)
    finally:
        if os.path.exists(path):
            os.unlink(path)
