"""Kill one rank mid-checkpoint, then restore on all ranks (SURVEY §4 "Distributed"; PAPER L283:
a checkpoint id is only usable once every peer holds it).

Two rank processes share cuda:0 (gloo carries the library's allreduce / allgather callbacks, as
in test_dp_gpu.py).  Iters 10 and 20 commit globally.  During iter 30 rank 1 SIGKILLs itself
(PCC_FAULT=header:3, before its COMPLETE header): rank 0 finishes 30 locally but no MIN over the
ranks ever reaches 30.  A fresh pair of processes must then agree on 20 and restore it bit-exactly
on both ranks (the allgather fan-out included), and the oracle reading both files must pick 20.
"""
import os
import subprocess
import sys

import numpy as np
import pytest

import oracle
from conftest import ROOT
from synth import config_tensors

pytestmark = [pytest.mark.gpu, pytest.mark.timeout(400)]
torch = pytest.importorskip("torch")
CB = 4 << 20

RANK = r"""
import datetime, os, sys
import numpy as np
sys.path.insert(0, sys.argv[5])
import torch
import torch.distributed as dist
rank, world, d, mode = int(sys.argv[1]), int(sys.argv[2]), sys.argv[3], sys.argv[4]
dist.init_process_group("gloo", rank=rank, world_size=world, timeout=datetime.timedelta(seconds=20))
import paper_conf_asplos_strati0k25_b200 as pcc
from synth import config_tensors, make_state, perturb_state, host_bytes
torch.cuda.set_device(0)
specs = config_tensors("c1")
ts = make_state(specs, "cuda", seed=51, it=0)

ck = pcc.PCCheck(os.path.join(d, f"r{rank}.pcc"), chunk_bytes=4 << 20, max_inflight=2,
                 flags=pcc.MAPFILE | pcc.FSYNC, rank=rank, world=world, **pcc.torch_collectives(dist))
ck.register(ts)
if mode == "crash":
    for it in (10, 20):
        perturb_state(ts, specs, 51, it)
        ck.wait(ck.checkpoint(it))
        assert ck.commit() == it
    np.save(os.path.join(d, f"s20_r{rank}.npy"), np.concatenate([host_bytes(t) for t in ts]))
    perturb_state(ts, specs, 51, 30)
    h = ck.checkpoint(30)
    ck.wait(h)  # rank 1 dies in here
    open(os.path.join(d, f"local30_r{rank}"), "w").close()
    ck.commit()  # the MIN can never see rank 1: gloo times out or the peer is gone
    sys.exit(9)
else:
    perturb_state(ts, specs, 51, 77)
    it, bad = ck.restore()
    ok = np.array_equal(np.concatenate([host_bytes(t) for t in ts]), np.load(os.path.join(d, f"s20_r{rank}.npy")))
    print("RESTORED", it, int(ok), len(bad), flush=True)
    ck.close()
"""


def _spawn(rank, d, mode, port, fault=None):
    env = dict(os.environ, MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    env.pop("PCC_FAULT", None)
    if fault:
        env["PCC_FAULT"] = fault
    return subprocess.Popen([sys.executable, "-c", RANK, str(rank), "2", d, mode, ROOT], env=env,
                            stdout=subprocess.PIPE, stderr=subprocess.PIPE, text=True)


@pytest.fixture
def shmdir(tmp_path):
    import shutil
    import tempfile
    d = tempfile.mkdtemp(dir="/dev/shm") if os.path.isdir("/dev/shm") else str(tmp_path)
    yield d
    shutil.rmtree(d, ignore_errors=True)


def test_kill_one_rank_mid_checkpoint_then_restore_all(shmdir):
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    port = 34500 + os.getpid() % 1000
    p0 = _spawn(0, shmdir, "crash", port)
    p1 = _spawn(1, shmdir, "crash", port, fault="header:3")
    out1, err1 = p1.communicate(timeout=240)
    assert p1.returncode == -9, (p1.returncode, err1[-3000:])  # SIGKILL inside iter 30
    try:
        out0, err0 = p0.communicate(timeout=120)  # its commit fails once the peer is gone
    except subprocess.TimeoutExpired:
        p0.kill()
        out0, err0 = p0.communicate()
    assert os.path.exists(os.path.join(shmdir, "local30_r0")), err0[-3000:]  # rank 0 holds 30 locally
    import paper_conf_asplos_strati0k25_b200 as pcc
    g0, l0 = pcc.latest(os.path.join(shmdir, "r0.pcc"))
    assert (g0, l0) == (20, 30)  # committed locally, never globally
    # a fresh pair restores: both ranks agree on 20 and get its bytes back
    procs = [_spawn(r, shmdir, "restore", port + 1) for r in range(2)]
    outs = [p.communicate(timeout=240) for p in procs]
    for p, (o, e) in zip(procs, outs):
        assert p.returncode == 0, e[-3000:]
        line = [x for x in o.splitlines() if x.startswith("RESTORED")][-1].split()
        assert line[1:] == ["20", "1", "0"], o
    specs = config_tensors("c1")
    paths = [os.path.join(shmdir, f"r{r}.pcc") for r in range(2)]
    rc, it, bad, outs = oracle.restore(paths, 3, [s.nbytes for s in specs], [s.code for s in specs], 256, CB)
    assert rc == 0 and it == 20
    assert np.array_equal(np.concatenate(outs), np.load(os.path.join(shmdir, "s20_r0.npy")))
