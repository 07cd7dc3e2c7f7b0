"""The NCCL-shaped C ABI on the GPU: program selection by size range (§6),
in-place / out-of-place forms, error codes, and CUDA-graph capture of a collective call."""
import numpy as np
import pytest

import synth
from oracle import irparse, mpi_ref, sim
from paper_conf_asplos_cowanmmsx23_b200 import programs as P

pytestmark = pytest.mark.gpu

R = 4


@pytest.fixture(scope="module")
def env():
    import torch
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    runtime.set_param("MSCCL_TIMEOUT_S", 10)
    comms = runtime.Comm.virtual(R, 0)
    yield torch, runtime, comms
    for c in comms:
        c.destroy()


def _call(runtime, comms, fn):
    with runtime.group():
        for q, c in enumerate(comms):
            fn(q, c)


def test_selection_by_size_range(env):
    torch, runtime, comms = env
    small = P.allpairs_allreduce(R)            # [0, 64 KiB)
    large = P.ring_allreduce(R, instances=2)   # [64 KiB, inf)
    ps = [(c.load(small.to_xml(), 0, 65536), c.load(large.to_xml(), 65536, 0)) for c in comms]
    try:
        for n, algo in ((1000, small), (100000, large)):
            xs = synth.inputs(R, n, "float32", "uniform")
            want = sim.simulate(irparse.parse(algo.to_xml()), xs, n, "float32")
            send = [torch.from_numpy(x).cuda() for x in xs]
            recv = [torch.empty_like(s) for s in send]
            _call(runtime, comms, lambda q, c: c.allreduce(send[q], recv[q]))
            torch.cuda.synchronize()
            for q in range(R):
                assert np.array_equal(recv[q].cpu().numpy().view(np.uint32), want[q].view(np.uint32))
        # no program for AllGather -> NoMatchingProgram, nothing launched
        x = torch.zeros(16, device="cuda")
        y = torch.zeros(16 * R, device="cuda")
        with pytest.raises(runtime.MscclError) as ei:
            comms[0].allgather(x, y)
        assert ei.value.code == 9
    finally:
        for c, (a, b) in zip(comms, ps):
            c.unload(a)
            c.unload(b)


def test_inplace_and_errors(env):
    torch, runtime, comms = env
    algo = P.ring_allreduce(R)
    ps = [c.load(algo.to_xml()) for c in comms]
    try:
        n = 5003
        xs = synth.inputs(R, n, "bfloat16", "intval")
        bufs = [torch.from_numpy(x.view(np.int16).copy()).cuda().view(torch.bfloat16) for x in xs]
        with pytest.raises(runtime.MscclError) as ei:   # out-of-place program, not aliassafe
            _call(runtime, comms, lambda q, c: c.allreduce(bufs[q], bufs[q]))
        assert ei.value.code == 5
        x = torch.zeros(64, device="cuda")
        with pytest.raises(runtime.MscclError) as ei:   # overlapping buffers
            comms[0].allreduce(x, x[8:].contiguous() if False else x.narrow(0, 8, 56), count=56)
        assert ei.value.code == 5
        # count == 0 is a no-op even outside a group
        comms[0].allreduce(x, torch.zeros(64, device="cuda"), count=0)
        # avg (4) is rejected
        import ctypes
        r = runtime.lib.mscclAllReduce(ctypes.c_void_p(x.data_ptr()), ctypes.c_void_p(x.data_ptr() + 1024), 4, 7, 4,
                                       comms[0].handle, None)
        assert r == 4
        # ranks sharing a GPU must be called together
        y = torch.zeros(64, device="cuda")
        with pytest.raises(runtime.MscclError) as ei:
            comms[0].allreduce(x, y)
        assert ei.value.code == 5
    finally:
        for c, p in zip(comms, ps):
            c.unload(p)


def test_inplace_program_called_out_of_place_gets_precopy(env):
    torch, runtime, comms = env
    algo = P.ring_allreduce(R, inplace=True)
    ps = [c.load(algo.to_xml()) for c in comms]
    try:
        n = 7777
        xs = synth.inputs(R, n, "float32", "intval")
        send = [torch.from_numpy(x).cuda() for x in xs]
        recv = [torch.full_like(s, -1) for s in send]
        _call(runtime, comms, lambda q, c: c.allreduce(send[q], recv[q]))
        torch.cuda.synchronize()
        ref = mpi_ref.allreduce(xs, "sum", "float32")[0].astype(np.float32)
        for q in range(R):
            assert np.array_equal(recv[q].cpu().numpy(), ref)
            assert np.array_equal(send[q].cpu().numpy(), xs[q])   # input untouched
        _call(runtime, comms, lambda q, c: c.allreduce(send[q], send[q]))  # true in-place
        torch.cuda.synchronize()
        for q in range(R):
            assert np.array_equal(send[q].cpu().numpy(), ref)
    finally:
        for c, p in zip(comms, ps):
            c.unload(p)


def test_cuda_graph_capture_and_replay(env):
    torch, runtime, comms = env
    algo = P.ring_allreduce(R, instances=2)
    ps = [c.load(algo.to_xml()) for c in comms]
    try:
        n = 65536
        xs = synth.inputs(R, n, "bfloat16", "uniform")
        want = sim.simulate(irparse.parse(algo.to_xml()), xs, n, "bfloat16")
        send = [torch.from_numpy(x.view(np.int16).copy()).cuda().view(torch.bfloat16) for x in xs]
        recv = [torch.empty_like(s) for s in send]
        _call(runtime, comms, lambda q, c: c.allreduce(send[q], recv[q]))  # warm-up (scratch etc.)
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            _call(runtime, comms, lambda q, c: c.allreduce(send[q], recv[q]))
        for _ in range(3):
            for r in recv:
                r.zero_()
            g.replay()
            torch.cuda.synchronize()
            for q in range(R):
                assert np.array_equal(recv[q].view(torch.int16).cpu().numpy().view(np.uint16), want[q])
    finally:
        for c, p in zip(comms, ps):
            c.unload(p)
