"""Host-side helpers of the Python binding (no GPU)."""
import pytest

torch = pytest.importorskip("torch")


def test_state_tensors_order_r11():
    """R11 order for SGD(momentum) and Adam, with and without fp32 masters; matches synth's
    model inventories' order (param, master, momentum | exp_avg, exp_avg_sq, step)."""
    import paper_conf_asplos_strati0k25_b200 as pcc
    m = torch.nn.Sequential(torch.nn.Linear(4, 3), torch.nn.Linear(3, 2))
    opt = torch.optim.SGD(m.parameters(), lr=0.1, momentum=0.9)
    m(torch.randn(2, 4)).sum().backward()
    opt.step()
    ts, names = pcc.state_tensors(opt)
    assert names == ["0.param", "0.momentum_buffer", "1.param", "1.momentum_buffer",
                     "2.param", "2.momentum_buffer", "3.param", "3.momentum_buffer"]
    ps = list(m.parameters())
    assert ts[0].data_ptr() == ps[0].data_ptr() and ts[1] is opt.state[ps[0]]["momentum_buffer"]
    opt = torch.optim.Adam(m.parameters(), lr=0.1, capturable=False)
    m(torch.randn(2, 4)).sum().backward()
    opt.step()
    ts, names = pcc.state_tensors(opt)  # CPU model: CPU step is on the params' device
    assert names[:4] == ["0.param", "0.exp_avg", "0.exp_avg_sq", "0.step"] and len(ts) == 16
    masters = {p: p.detach().double() for p in ps}
    ts, names = pcc.state_tensors(opt, masters)
    assert names[:5] == ["0.param", "0.master", "0.exp_avg", "0.exp_avg_sq", "0.step"]
    assert ts[1] is masters[ps[0]]


def test_state_tensors_rejects_host_state_of_device_params():
    import paper_conf_asplos_strati0k25_b200 as pcc

    class FakeOpt:
        def __init__(self, p):
            self.param_groups = [{"params": [p]}]
            self.state = {p: {"exp_avg": torch.zeros(2, device="meta"), "step": 3}}
    p = torch.nn.Parameter(torch.zeros(2, device="meta"))
    with pytest.raises(ValueError):
        pcc.state_tensors(FakeOpt(p))


def _coll_worker(rank, world, port, q):
    import os
    import numpy as np
    import torch.distributed as dist
    import paper_conf_asplos_strati0k25_b200 as pcc
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        coll = pcc.torch_collectives(dist)
        assert coll["allreduce"]([rank + 5, -rank], True) == [world + 4, 0]
        assert coll["allreduce"]([rank + 5, -rank], False) == [5, -(world - 1)]
        n = 1 << 20  # one MiB per rank, written in place into the receive view
        send = np.full(n, 17 + rank, dtype=np.uint8)
        recv = np.zeros(world * n, dtype=np.uint8)
        coll["allgather"](send, recv)
        ok = all((recv[r * n:(r + 1) * n] == 17 + r).all() for r in range(world))
        coll["allgather"](np.empty(0, np.uint8), np.empty(0, np.uint8))  # zero bytes per rank
        q.put((rank, bool(ok)))
    finally:
        dist.destroy_process_group()


def test_torch_collectives_gloo_world2():
    """The zero-copy gloo adapter the DP tests and the binding use for caller collectives:
    allreduce MIN/MAX and an in-place rank-ordered allgather into the receive view."""
    import os
    import torch.multiprocessing as mp
    port = 31000 + os.getpid() % 2000
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_coll_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    for p in ps:
        p.join(120)
        assert p.exitcode == 0
    assert sorted(q.get(timeout=10) for _ in range(2)) == [(0, True), (1, True)]
