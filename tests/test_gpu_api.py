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
        _call(runtime, comms, lambda q, c: c.allreduce(send[q], recv[q]))  # warm-up
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


@pytest.mark.parametrize("make", ["allpairs", "oneshot"])
def test_first_call_of_fresh_program_captured_in_graph(env, make):
    """SURVEY §8(b) Ownership: a program loaded with maxBytes has its scratch pre-sized, so
    the FIRST call after mscclLoadProgram can be captured in a CUDA graph (no allocation, no
    host sync) and the replays are bit-exact with the oracle."""
    torch, runtime, comms = env
    algo = P.allpairs_allreduce(R, protocol="Simple") if make == "allpairs" else P.oneshot_allreduce(R, protocol="LL")
    n = 12289
    ps = [c.load(algo.to_xml(), 0, 1 << 20) for c in comms]
    try:
        xs = synth.inputs(R, n, "float16", "uniform")
        want = sim.simulate(irparse.parse(algo.to_xml()), xs, n, "float16")
        send = [torch.from_numpy(x.view(np.int16).copy()).cuda().view(torch.float16) for x in xs]
        recv = [torch.empty_like(s) for s in send]
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            _call(runtime, comms, lambda q, c: c.allreduce(send[q], recv[q]))
        for _ in range(2):
            for r in recv:
                r.zero_()
            g.replay()
            torch.cuda.synchronize()
            for q in range(R):
                assert np.array_equal(recv[q].view(torch.int16).cpu().numpy().view(np.uint16), want[q].view(np.uint16))
    finally:
        for c, p in zip(comms, ps):
            c.unload(p)


def test_scratch_growth_during_capture_is_refused(env):
    """A program loaded without maxBytes grows scratch on demand; if that would happen while
    the stream is being captured the call returns InvalidUsage (nothing is captured), and
    after one uncaptured call of that size capture works."""
    torch, runtime, comms = env
    algo = P.allpairs_allreduce(R, protocol="Simple")
    ps = [c.load(algo.to_xml()) for c in comms]
    try:
        n = 50001
        xs = synth.inputs(R, n, "float32", "uniform")
        want = sim.simulate(irparse.parse(algo.to_xml()), xs, n, "float32")
        send = [torch.from_numpy(x).cuda() for x in xs]
        recv = [torch.empty_like(s) for s in send]
        torch.cuda.synchronize()
        s = torch.cuda.Stream()
        g = torch.cuda.CUDAGraph()
        with pytest.raises(runtime.MscclError) as ei:
            with torch.cuda.graph(g, stream=s):
                _call(runtime, comms, lambda q, c: c.allreduce(send[q], recv[q]))
        assert ei.value.code == 5
        torch.cuda.synchronize()
        _call(runtime, comms, lambda q, c: c.allreduce(send[q], recv[q]))   # grows scratch
        torch.cuda.synchronize()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g):
            _call(runtime, comms, lambda q, c: c.allreduce(send[q], recv[q]))
        for r in recv:
            r.zero_()
        g.replay()
        torch.cuda.synchronize()
        for q in range(R):
            assert np.array_equal(recv[q].cpu().numpy().view(np.uint32), want[q].view(np.uint32))
    finally:
        for c, p in zip(comms, ps):
            c.unload(p)


def test_two_calls_on_one_comm_in_one_group_rejected(env):
    """two collectives on the same communicator inside one group would share its
    connection counters and semaphores in one grid; the launch is refused."""
    torch, runtime, comms = env
    algo = P.ring_allreduce(R)
    ps = [c.load(algo.to_xml()) for c in comms]
    try:
        x = torch.zeros(4096, device="cuda")
        ys = [torch.zeros(4096, device="cuda") for _ in range(R + 1)]
        with pytest.raises(runtime.MscclError) as ei:
            with runtime.group():
                for q, c in enumerate(comms):
                    c.allreduce(x, ys[q])
                comms[0].allreduce(x, ys[R])
        assert ei.value.code == 5
    finally:
        torch.cuda.synchronize()
        for c, p in zip(comms, ps):
            c.unload(p)


def test_aliassafe_inplace_call_disables_direct_placement(env):
    """an out-of-place program marked aliassafe may be called in place; the
    launch then runs without direct placement (its analysis assumes distinct in/out) and the
    result equals the out-of-place result bit for bit."""
    torch, runtime, comms = env
    ir = P.ring_allreduce(R, instances=2).to_xml().replace("<algo ", '<algo aliassafe="1" ', 1)
    ps = [c.load(ir) for c in comms]
    try:
        n = 40000
        xs = synth.inputs(R, n, "float32", "uniform")
        want = sim.simulate(irparse.parse(ir), xs, n, "float32")
        bufs = [torch.from_numpy(x).cuda() for x in xs]
        _call(runtime, comms, lambda q, c: c.allreduce(bufs[q], bufs[q]))
        torch.cuda.synchronize()
        for q in range(R):
            assert np.array_equal(bufs[q].cpu().numpy().view(np.uint32), want[q].view(np.uint32))
    finally:
        for c, p in zip(comms, ps):
            c.unload(p)


def test_v9_rechecked_once_per_pipeline_depth(env):
    """Reading R24: the loader verified deadlock freedom over 2
    pipeline iterations; the first launch with a deeper pipeline re-runs V9 at its real depth
    I, once per (program, I) -- a second call of the same size is not re-checked, a larger
    size is. One-launch direct placement counts too (mscclCommGetStats)."""
    torch, runtime, comms = env
    algo = P.ring_allreduce(R, instances=2)
    ps = [c.load(algo.to_xml()) for c in comms]
    try:
        slot = runtime.get_param("MSCCL_SLOT_BYTES")
        def run(n):
            x = [torch.ones(n, device="cuda") for _ in comms]
            y = [torch.empty_like(t) for t in x]
            _call(runtime, comms, lambda q, c: c.allreduce(x[q], y[q]))
            torch.cuda.synchronize()
            assert all(bool((t == R).all()) for t in y)
        s0 = comms[0].stats()
        n1 = (slot // 4) * R * 2 * 3          # 3 tiles per chunk (fp32)
        run(n1)
        s1 = comms[0].stats()
        assert s1["depth_checks"] == s0["depth_checks"] + 1
        assert s1["launches_direct1"] == s0["launches_direct1"] + 1
        run(n1)
        assert comms[0].stats()["depth_checks"] == s1["depth_checks"]
        run(n1 * 2)
        assert comms[0].stats()["depth_checks"] == s1["depth_checks"] + 1
    finally:
        for c, p_ in zip(comms, ps):
            c.unload(p_)


def _range_sizes(lo, hi, w, cap=8 << 20):
    """byte sizes that probe one [lo, hi) range: its start, a ragged size inside, its end"""
    out = []
    if lo > 0:
        out.append(lo)
    out.append(min(lo + 6 * w + 2 * w, cap) if hi == 0 else min(lo + (hi - lo) // 3 + 2 * w, cap))
    if hi:
        out.append(min(hi - 2 * w, cap))
    return sorted({(b // w) * w for b in out if b >= w})


@pytest.mark.parametrize("which", ["tuned_allreduce", "tuned_allreduce_multimem"])
def test_tuned_allreduce_sets_through_the_public_api(which):
    """The size-range program sets (§6) as a user runs them: every program loaded
    with its range, mscclAllReduce at each range's start, inside and end (8 ranks, bf16); the
    result equals, bit for bit, the oracle running the program the range selects."""
    import torch
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    W = 8
    sets = getattr(P, which)(W)
    comms = runtime.Comm.virtual(W, 0)
    try:
        for c in comms:
            for algo, lo, hi in sets:
                c.load(algo.to_xml(), lo, hi)
        for algo, lo, hi in sets:
            for nbytes in _range_sizes(lo, hi, 2):
                n = nbytes // 2
                xs = synth.inputs(W, n, "bfloat16", "uniform", seed=nbytes)
                want = sim.simulate(irparse.parse(algo.to_xml()), xs, n, "bfloat16", "sum")
                send = [torch.from_numpy(x.view(np.int16).copy()).cuda().view(torch.bfloat16) for x in xs]
                recv = [torch.empty_like(s) for s in send]
                _call(runtime, comms, lambda q, c: c.allreduce(send[q], recv[q]))
                torch.cuda.synchronize()
                for q in range(W):
                    got = recv[q].view(torch.int16).cpu().numpy().view(np.uint16)
                    assert np.array_equal(got, want[q].view(np.uint16)), (which, algo.name, nbytes, q)
    finally:
        for c in comms:
            c.destroy()


def test_tuned_alltoall_set_through_the_public_api():
    """mscclAllToAll with the AllToAll size-range set (selection bytes = per-peer count * w):
    exact permutation at each range's start, inside and end."""
    import torch
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    W = 8
    sets = P.tuned_alltoall(W)
    comms = runtime.Comm.virtual(W, 0)
    try:
        for c in comms:
            for algo, lo, hi in sets:
                c.load(algo.to_xml(), lo, hi)
        for algo, lo, hi in sets:
            for nbytes in _range_sizes(lo, hi, 4, cap=1 << 20):
                n = nbytes // 4   # per-peer count
                xs = synth.inputs(W, W * n, "int32", "pattern")
                send = [torch.from_numpy(x.copy()).cuda() for x in xs]
                recv = [torch.empty_like(s) for s in send]
                _call(runtime, comms, lambda q, c: c.alltoall(send[q], recv[q]))
                torch.cuda.synchronize()
                for q, e in enumerate(mpi_ref.alltoall(xs, n)):
                    assert np.array_equal(recv[q].cpu().numpy(), e), (algo.name, nbytes, q)
    finally:
        for c in comms:
            c.destroy()


@pytest.mark.parametrize("make", ["allpairs", "oneshot", "hier"])
def test_semaphores_across_the_generation_wrap(make):
    """Programs with cross-thread-block dependencies launched across 2^24 launches of their
    thread blocks (the generation field of a semaphore wraps, reading R4): every launch
    bit-exact. With a plain >= on the semaphore word the launch right after the wrap saw the
    previous launch's (larger) value as done and read its inputs too early."""
    import torch
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    W = 4
    algo = {"allpairs": lambda: P.allpairs_allreduce(W, protocol="Simple"),
            "oneshot": lambda: P.oneshot_allreduce(W, protocol="Simple"),
            "hier": lambda: P.hierarchical_allreduce(2, 2)}[make]()
    comms = runtime.Comm.virtual(W, 0)
    try:
        progs = [c.load(algo.to_xml()) for c in comms]
        for p in progs:
            p.set_generation((1 << 24) - 3)
        for it in range(6):
            n = 200003 + it
            xs = synth.inputs(W, n, "float32", "uniform", seed=it)
            want = sim.simulate(irparse.parse(algo.to_xml()), xs, n, "float32")
            send = [torch.from_numpy(x).cuda() for x in xs]
            recv = [torch.empty_like(s) for s in send]
            _call(runtime, comms, lambda q, c: c.run(progs[q], send[q], recv[q], n))
            torch.cuda.synchronize()
            for q in range(W):
                assert np.array_equal(recv[q].cpu().numpy().view(np.uint32), want[q].view(np.uint32)), (it, q)
    finally:
        for c in comms:
            c.destroy()
