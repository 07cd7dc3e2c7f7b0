"""One process per rank (mscclCommInitRank + CUDA IPC handle exchange + mscclCommConnect):
the code path of the one-process-per-GPU deployment, run here
with 2, 4 and 8 processes sharing the single available GPU. Their kernels time-slice, so
only small messages are used. Every process opens its peers' regions through CUDA IPC and
runs the interpreter with system-scope flags.

Every shipped program family runs under Simple, LL and LL128: ring, all-pairs, one-shot,
hierarchical, two-step AllToAll, AllGather and ReduceScatter. Simple cases run twice: once
through the receiver-side FIFO only, and once with the send/receive buffers registered
(mscclCommRegister), which turns on cross-launch direct placement. In that mode a sender
waits for the receiver's per-launch ready line, then stores straight into the receiver's
IPC-mapped buffer (reading R15b). Every result is compared bit-exactly with the oracle.
"""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu

# Ranks that wait on one another, run as separate processes time-slicing one GPU, can raise
# Xid 109 (context-switch timeout) on this driver (B200_PROFILING.md). The tests that launch
# such kernels ran green in this round's explicit runs (profiles/r02/gpu_tests_final.log); the
# default GPU suite covers the same cross-launch device code with every rank co-resident in one
# launch instead (tests/test_gpu_cross_launch.py). Set MSCCL_MULTIPROC_GPU=1 to run them on a
# GPU box where that is safe. The Connect test below launches no kernel and always runs.
spinning = pytest.mark.skipif(os.environ.get("MSCCL_MULTIPROC_GPU") != "1",
                              reason="separate processes spinning on one GPU (Xid 109 risk); "
                                     "set MSCCL_MULTIPROC_GPU=1; covered by test_gpu_cross_launch.py")


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _algo(name, W, proto):
    from paper_conf_asplos_cowanmmsx23_b200 import programs as P
    if name == "ring":
        return P.ring_allreduce(W, protocol=proto)
    if name == "ring_i2":
        return P.ring_allreduce(W, instances=2, protocol=proto)
    if name == "ring_ch":
        return P.ring_allreduce(W, channels=W, protocol=proto)
    if name == "ring_inplace":
        return P.ring_allreduce(W, protocol=proto, inplace=True)
    if name == "allpairs":
        return P.allpairs_allreduce(W, protocol=proto)
    if name == "oneshot":
        return P.oneshot_allreduce(W, protocol=proto)
    if name == "hier":
        return P.hierarchical_allreduce(2, W // 2, protocol=proto)
    if name == "a2a":
        return P.alltoall_twostep(1, W, protocol=proto)
    if name == "a2a_2step":
        return P.alltoall_twostep(2, W // 2, protocol=proto)
    if name == "allgather":
        return P.ring_allgather(W, 1, 2, protocol=proto)
    if name == "reducescatter":
        return P.ring_reducescatter(W, 1, 2, protocol=proto)
    if name == "nvls_ar":
        return P.nvls_allreduce(W, 2)
    if name == "nvls_rs":
        return P.nvls_reducescatter(W, 2)
    if name == "nvls_ag":
        return P.nvls_allgather(W, 2)
    if name == "ring_mm":
        return P.ring_rs_multimem_ag_allreduce(W, 2)
    raise KeyError(name)


# (program, protocol, dtype, op, n per block, register buffers)
CASES = [
    ("ring", "Simple", "float32", "sum", 20003, False),
    ("ring", "Simple", "float32", "sum", 20003, True),
    ("ring_i2", "Simple", "bfloat16", "sum", 30001, True),
    ("ring_inplace", "Simple", "float32", "sum", 9001, True),
    ("ring", "LL", "bfloat16", "sum", 3001, False),
    ("ring", "LL128", "float16", "sum", 9001, False),
    ("ring_ch", "Simple", "int32", "max", 12345, True),
    ("allpairs", "Simple", "float32", "sum", 8191, True),
    ("allpairs", "LL", "float16", "sum", 2049, False),
    ("oneshot", "LL", "bfloat16", "sum", 512, False),
    ("oneshot", "Simple", "float32", "min", 4099, True),
    ("hier", "Simple", "float32", "sum", 16001, True),
    ("hier", "LL128", "int32", "sum", 5003, False),
    ("a2a", "Simple", "bfloat16", None, 6007, False),
    ("a2a", "Simple", "bfloat16", None, 6007, True),
    ("a2a_2step", "Simple", "int32", None, 2001, True),
    ("a2a", "LL", "int32", None, 777, False),
    ("allgather", "Simple", "int32", None, 7001, True),
    ("allgather", "LL128", "uint8", None, 3333, False),
    ("reducescatter", "Simple", "float32", "sum", 5001, True),
    ("reducescatter", "LL", "float32", "prod", 1201, False),
    # multimem (NVLS) programs across processes: group barrier + registered buffers (reading R23)
    ("nvls_ar", "Simple", "bfloat16", "sum", 20011, True),
    ("nvls_ar", "Simple", "int32", "max", 7001, True),
    ("nvls_rs", "Simple", "float32", "sum", 9001, True),
    ("nvls_ag", "Simple", "int32", None, 5003, True),
    ("ring_mm", "Simple", "float32", "sum", 12007, True),
]


# registered Simple cases whose programs place messages directly into in/out buffers
DIRECT_EXPECTED = {"ring", "ring_i2", "ring_ch", "allpairs", "a2a", "a2a_2step", "allgather"}


def _inputs(name, W, n, dtype):
    import synth
    from oracle import geometry
    algo = _algo(name, W, "Simple")
    coll = {"a2a": "alltoall", "a2a_2step": "alltoall", "allgather": "allgather", "nvls_ag": "allgather",
            "reducescatter": "reducescatter", "nvls_rs": "reducescatter"}.get(name, "allreduce")
    elems = geometry.buffer_elems(coll, "i", W, n)
    del algo
    dist = "pattern" if coll in ("alltoall", "allgather") else ("uniform" if dtype.startswith(("float", "bf"))
                                                                  else "int")
    if dtype == "uint8":
        dist = "pattern"
    return synth.inputs(W, elems, dtype, dist), geometry.buffer_elems(coll, "o", W, n)


def _worker(rank, world, port, q, cases):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    out = []
    try:
        from paper_conf_asplos_cowanmmsx23_b200 import dist as mdist
        from paper_conf_asplos_cowanmmsx23_b200 import runtime
        runtime.set_param("MSCCL_TIMEOUT_S", 120)
        runtime.set_param("MSCCL_SLOT_BYTES", 16384)
        runtime.set_param("MSCCL_LL_SLOT_BYTES", 16384)
        runtime.set_param("MSCCL_LL128_SLOT_BYTES", 16384)
        runtime.set_param("MSCCL_MAX_CHANNELS", 8)
        runtime.set_param("MSCCL_THREADS", 128)
        comm = mdist.init_from_process_group(0)
        for ci, (name, proto, dtype, op, n, reg) in enumerate(cases):
            algo = _algo(name, world, proto)
            prog = comm.load(algo.to_xml())
            xs, out_elems = _inputs(name, world, n, dtype)
            x = torch.from_numpy(xs[rank].view(np.uint8).copy()).cuda()
            inplace = name == "ring_inplace"
            y = x if inplace else torch.full((out_elems * xs[0].itemsize,), 0xA5, dtype=torch.uint8, device="cuda")
            regs = []
            if reg:
                regs = [mdist.register(comm, x)] + ([] if inplace else [mdist.register(comm, y)])
            h0 = comm.stats()["cross_direct_handshakes"]
            for _ in range(2):   # twice: the second launch reuses the ready lines / registrations
                if inplace:
                    x.copy_(torch.from_numpy(xs[rank].view(np.uint8).copy()).cuda())
                comm.run(prog, x, y, n, op=op or "sum", dtype=dtype)
                torch.cuda.synchronize()
            res = y.cpu().numpy().copy()
            hs = comm.stats()["cross_direct_handshakes"] - h0
            dist.barrier()
            for r_ in regs:
                r_.deregister()
            comm.unload(prog)
            out.append((ci, res, comm.async_error(), hs))
            dist.barrier()
        q.put((rank, out))
        dist.barrier()
        comm.destroy()
    except Exception as e:  # report, never hang the parent
        import traceback
        q.put((rank, "%r\n%s" % (e, traceback.format_exc())))
    finally:
        dist.destroy_process_group()


def _expected(name, W, proto, dtype, op, n):
    from oracle import irparse, sim
    xs, _ = _inputs(name, W, n, dtype)
    algo = irparse.parse(_algo(name, W, proto).to_xml())
    return sim.simulate(algo, xs, n, dtype, op or "sum")


def _run_world(world, cases, timeout):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, cases)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    try:
        for _ in range(world):
            r, out = q.get(timeout=timeout)
            res[r] = out
    finally:
        for p in procs:
            p.join(timeout=60)
            if p.is_alive():
                p.kill()
    for r in range(world):
        assert not isinstance(res[r], str), res[r]
    for ci, (name, proto, dtype, op, n, reg) in enumerate(cases):
        want = _expected(name, world, proto, dtype, op, n)
        handshakes = 0
        for r in range(world):
            k, got, err, hs = res[r][ci]
            assert k == ci and err == 0, (name, proto, r, err)
            w = np.ascontiguousarray(want[r]).view(np.uint8)
            assert np.array_equal(got[:w.size], w), (name, proto, dtype, reg, "rank", r)
            handshakes += hs
        # device-side evidence of cross-launch direct placement (reading R15b): senders found
        # a registered destination exactly when the buffers were registered
        if not reg or proto != "Simple" or name.startswith("nvls") or name == "ring_mm":
            assert handshakes == 0, (name, proto, handshakes)
        elif name in DIRECT_EXPECTED:
            assert handshakes > 0, (name, proto, handshakes)


@spinning
@pytest.mark.parametrize("world", [2, 4, 8])
def test_processes_ipc_all_programs(world):
    cases = [c for c in CASES if not (c[0] in ("hier", "a2a_2step") and world < 4)]
    _run_world(world, cases, timeout=900)


def _silent_peer_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_asplos_cowanmmsx23_b200 import dist as mdist
        from paper_conf_asplos_cowanmmsx23_b200 import programs, runtime
        runtime.set_param("MSCCL_TIMEOUT_S", 3)
        runtime.set_param("MSCCL_SLOT_BYTES", 16384)
        runtime.set_param("MSCCL_MAX_CHANNELS", 2)
        runtime.set_param("MSCCL_THREADS", 64)
        comm = mdist.init_from_process_group(0)
        comm.load(programs.ring_allreduce(world).to_xml())
        res = None
        if rank == 0:  # rank 1 never joins the collective: rank 0's kernel must not hang
            x = torch.ones(4096, device="cuda")
            y = torch.empty_like(x)
            comm.allreduce(x, y)
            torch.cuda.synchronize()
            err = comm.async_error()
            try:
                comm.allreduce(x, y)
                again = "no error"
            except runtime.MscclError as e:
                again = e.code
            res = (err, again)
        dist.barrier()
        q.put((rank, res))
    except Exception as e:
        q.put((rank, repr(e)))
    finally:
        dist.destroy_process_group()


@spinning
def test_watchdog_turns_a_missing_peer_into_an_error():
    """A peer that never launches: the spin waits time out (MSCCL_TIMEOUT_S), the kernel
    exits, and the communicator reports mscclRemoteError (sticky) instead of hanging."""
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_silent_peer_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=180) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert res[0] == (6, 6), res  # async error RemoteError, and the next call refuses


def _mismatch_worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_asplos_cowanmmsx23_b200 import dist as mdist
        from paper_conf_asplos_cowanmmsx23_b200 import runtime
        runtime.set_param("MSCCL_SLOTS", 4 if rank == 0 else 2)   # ranks disagree
        runtime.set_param("MSCCL_MAX_CHANNELS", 2)
        try:
            mdist.init_from_process_group(0)
            q.put((rank, "connected"))
        except runtime.MscclError as e:
            q.put((rank, (e.code, "MSCCL_SLOTS" in str(e) or "region size" in str(e))))
    finally:
        dist.destroy_process_group()


def test_connect_rejects_mismatched_parameters():
    """mscclCommConnect compares the slot geometry of every peer."""
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_mismatch_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=180) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
    assert res[0] == (5, True) and res[1] == (5, True), res


SEQUENCE = [("ring", "Simple", "float32", "sum", 30001, True), ("a2a", "Simple", "bfloat16", None, 4003, True),
            ("ring", "LL", "bfloat16", "sum", 2001, False), ("nvls_ar", "Simple", "bfloat16", "sum", 9001, True),
            ("allgather", "Simple", "int32", None, 5001, True), ("ring", "LL128", "float16", "sum", 7001, False),
            ("ring_i2", "Simple", "bfloat16", "sum", 40001, False), ("ring_mm", "Simple", "float32", "sum", 8001, True)]


def _sequence_worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_asplos_cowanmmsx23_b200 import dist as mdist
        from paper_conf_asplos_cowanmmsx23_b200 import runtime
        runtime.set_param("MSCCL_TIMEOUT_S", 120)
        for k in ("MSCCL_SLOT_BYTES", "MSCCL_LL_SLOT_BYTES", "MSCCL_LL128_SLOT_BYTES"):
            runtime.set_param(k, 16384)
        runtime.set_param("MSCCL_MAX_CHANNELS", 8)
        runtime.set_param("MSCCL_THREADS", 128)
        comm = mdist.init_from_process_group(0)
        progs = [comm.load(_algo(name, world, proto).to_xml()) for name, proto, *_ in SEQUENCE]
        bufs = []
        for name, proto, dtype, op, n, reg in SEQUENCE:
            xs, out_elems = _inputs(name, world, n, dtype)
            x = torch.from_numpy(xs[rank].view(np.uint8).copy()).cuda()
            y = torch.full((out_elems * xs[0].itemsize,), 0xA5, dtype=torch.uint8, device="cuda")
            regs = [mdist.register(comm, x), mdist.register(comm, y)] if reg else []
            bufs.append((x, y, regs))
        for rep in range(2):   # every program back to back on one stream, no host sync in between
            for (name, proto, dtype, op, n, reg), p, (x, y, _) in zip(SEQUENCE, progs, bufs):
                comm.run(p, x, y, n, op=op or "sum", dtype=dtype)
        torch.cuda.synchronize()
        out = [y.cpu().numpy().copy() for _, y, _ in bufs]
        dist.barrier()
        for _, _, regs in bufs:
            for r_ in regs:
                r_.deregister()
        q.put((rank, out, comm.async_error()))
        dist.barrier()
        comm.destroy()
    except Exception as e:
        import traceback
        q.put((rank, "%r\n%s" % (e, traceback.format_exc()), -1))
    finally:
        dist.destroy_process_group()


@spinning
def test_mixed_program_sequence_four_processes():
    """Eight different programs -- Simple with and without registered buffers, LL, LL128,
    multimem, and a mixed program -- run back to back twice on one stream per process. The
    per-connection launch ordinals, the ready lines, the multimem epochs and the
    per-protocol FIFOs must stay consistent across every kind of launch (R15b, R20, R23).
    Every output is bit-exact with the oracle."""
    world = 4
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_sequence_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    try:
        for _ in range(world):
            r, out, err = q.get(timeout=900)
            res[r] = (out, err)
    finally:
        for p in procs:
            p.join(timeout=60)
            if p.is_alive():
                p.kill()
    for r in range(world):
        assert not isinstance(res[r][0], str), res[r][0]
        assert res[r][1] == 0
    for k, (name, proto, dtype, op, n, reg) in enumerate(SEQUENCE):
        want = _expected(name, world, proto, dtype, op, n)
        for r in range(world):
            w = np.ascontiguousarray(want[r]).view(np.uint8)
            assert np.array_equal(res[r][0][k][:w.size], w), (name, proto, r)
