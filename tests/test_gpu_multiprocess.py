"""One process per rank (mscclCommInitRank + CUDA IPC handle exchange + mscclCommConnect)
on the single available GPU: both ranks' processes open each other's regions through CUDA
IPC and run the interpreter with system-scope flags, exactly the code path of the
multi-GPU deployment. The two processes' kernels share the GPU by time slicing, so only
small messages are used; results are checked bit-exactly against the oracle.
"""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q, prog_name, n):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import synth
        from paper_conf_asplos_cowanmmsx23_b200 import dist as mdist
        from paper_conf_asplos_cowanmmsx23_b200 import programs, runtime
        runtime.set_param("MSCCL_TIMEOUT_S", 60)
        runtime.set_param("MSCCL_SLOT_BYTES", 16384)
        runtime.set_param("MSCCL_MAX_CHANNELS", 4)
        runtime.set_param("MSCCL_THREADS", 128)
        comm = mdist.init_from_process_group(0)
        algo = {"ring": programs.ring_allreduce(world), "allpairs": programs.allpairs_allreduce(world),
                "ring_LL128": programs.ring_allreduce(world, protocol="LL128")}[prog_name]
        comm.load(algo.to_xml())
        x = torch.from_numpy(synth.rank_input(rank, n, "float32", "uniform")).cuda()
        y = torch.empty_like(x)
        comm.allreduce(x, y)
        torch.cuda.synchronize()
        q.put((rank, y.cpu().numpy(), comm.async_error()))
        dist.barrier()
        comm.destroy()
    except Exception as e:  # report, never hang the parent
        q.put((rank, repr(e), -1))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("prog_name", ["ring", "allpairs", "ring_LL128"])
def test_two_processes_ipc(prog_name):
    from oracle import irparse, sim
    from paper_conf_asplos_cowanmmsx23_b200 import programs
    import synth
    world, n = 2, 20000 + 3
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q, prog_name, n)) for r in range(world)]
    for p in procs:
        p.start()
    res = {}
    for _ in range(world):
        r, y, err = q.get(timeout=240)
        res[r] = (y, err)
    for p in procs:
        p.join(timeout=60)
    algo = {"ring": programs.ring_allreduce(world), "allpairs": programs.allpairs_allreduce(world),
            "ring_LL128": programs.ring_allreduce(world, protocol="LL128")}[prog_name]
    xs = synth.inputs(world, n, "float32", "uniform")
    want = sim.simulate(irparse.parse(algo.to_xml()), xs, n, "float32")
    for r in range(world):
        y, err = res[r]
        assert err == 0, y
        assert np.array_equal(np.asarray(y).view(np.uint32), want[r].view(np.uint32))


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
