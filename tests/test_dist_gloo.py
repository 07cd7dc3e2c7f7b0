"""Multi-process host logic on CPU: world size 2 over gloo (127.0.0.1).

The one-process-per-GPU mode exchanges each rank's region handle (CUDA IPC bytes) over a
torch.distributed group and connects. Here the communicator is a stand-in that records
what it receives, so the exchange, ordering and validation run without a GPU. The
per-rank program-selection rules are exercised on the same two processes through the
DSL + C++ validator (identical programs must validate identically on every rank).
"""
import os
import socket

import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class FakeComm:
    def __init__(self, rank):
        self.rank = rank
        self.got = None

    def export_handle(self):
        return bytes([self.rank]) * 128

    def connect(self, handles):
        self.got = handles


def _worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_asplos_cowanmmsx23_b200 import dist as mdist
        from paper_conf_asplos_cowanmmsx23_b200 import programs, runtime
        c = mdist.connect(FakeComm(rank))
        ok_order = [h[0] for h in c.got] == list(range(world)) and all(len(h) == 128 for h in c.got)
        ir = programs.ring_allreduce(world, instances=2).to_xml()
        verdicts = [None] * world
        dist.all_gather_object(verdicts, runtime.validate(ir, world)[0])
        q.put((rank, ok_order, verdicts))
    finally:
        dist.destroy_process_group()


def test_handle_exchange_two_ranks():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, ok_order, verdicts in res:
        assert ok_order
        assert verdicts == [True, True]


def test_inconsistent_handles_rejected(monkeypatch):
    from paper_conf_asplos_cowanmmsx23_b200 import dist as mdist

    class D:
        @staticmethod
        def get_world_size(group=None):
            return 2

        @staticmethod
        def all_gather_object(out, obj, group=None):
            out[0] = obj
            out[1] = obj[:10]

    import torch
    monkeypatch.setattr(torch, "distributed", D, raising=False)
    import sys
    monkeypatch.setitem(sys.modules, "torch.distributed", D)
    with pytest.raises(RuntimeError):
        mdist.exchange_handles(b"x" * 128)


class FakeReg:
    def __init__(self, rank):
        self.rank = rank
        self.got = None

    def export(self):
        return bytes([0x40 + self.rank]) * 128

    def connect(self, descs):
        self.got = descs


class FakeRegComm(FakeComm):
    def register(self, tensor):
        self.reg = FakeReg(self.rank)
        self.reg.tensor = tensor
        return self.reg


def _register_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_asplos_cowanmmsx23_b200 import dist as mdist
        c = FakeRegComm(rank)
        reg = mdist.register(c, torch.zeros(4))
        q.put((rank, [d[0] - 0x40 for d in reg.got], all(len(d) == 128 for d in reg.got)))
    finally:
        dist.destroy_process_group()


def test_buffer_registration_exchange_two_ranks():
    """dist.register (reading R15b): every rank's registration descriptor reaches every rank
    in rank order (mscclRegConnect's contract), over a real world-size-2 gloo group."""
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_register_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=120) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, order, sizes in res:
        assert order == [0, 1] and sizes
