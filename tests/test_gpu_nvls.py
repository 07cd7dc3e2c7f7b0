"""GPU parity of the multimem (NVLS) ops (reading R23) on virtual
ranks: every rank of the group is in one launch, so the interpreter reaches every rank's
buffer directly (the unicast form of multimem ld_reduce / st). Outputs are compared bit for
bit with the oracle simulator (fp32 accumulation and one rounding for fp16 / bf16 sums,
ascending-rank fold), and with the MPI definitions on integer-valued inputs. The
cross-process form (group barrier, registered buffers) is covered by
tests/test_gpu_multiprocess.py."""
import numpy as np
import pytest

import synth
from oracle import irparse, mpi_ref, sim
from paper_conf_asplos_cowanmmsx23_b200 import programs as P

pytestmark = pytest.mark.gpu


def _run(algo, xs, n, dtype, op="sum", out_elems=None):
    import gpu_util
    return gpu_util.run_program(algo.to_xml(), xs, n, dtype, op, out_elems=out_elems)


@pytest.mark.parametrize("R", [2, 4, 8])
@pytest.mark.parametrize("r", [1, 2, 4])
@pytest.mark.parametrize("dtype,op", [("bfloat16", "sum"), ("float16", "sum"), ("float32", "sum"),
                                      ("float32", "max"), ("int32", "sum"), ("bfloat16", "min"),
                                      ("float64", "sum"), ("uint8", "max")])
def test_nvls_allreduce_bit_exact(R, r, dtype, op):
    n = 4097 * r + 13
    dist = "uniform" if dtype.startswith(("float", "bf")) else "int"
    xs = synth.inputs(R, n, dtype, dist)
    algo = P.nvls_allreduce(R, r)
    want = sim.simulate(irparse.parse(algo.to_xml()), xs, n, dtype, op)
    got = _run(algo, xs, n, dtype, op)
    for g, w in zip(got, want):
        assert np.array_equal(np.asarray(g).view(np.uint8), np.asarray(w).view(np.uint8))


@pytest.mark.parametrize("R", [4, 8])
def test_nvls_allreduce_integer_valued_matches_mpi(R):
    n = 100003
    xs = synth.inputs(R, n, "bfloat16", "intval")
    got = _run(P.nvls_allreduce(R, 2), xs, n, "bfloat16", "sum")
    from oracle import numerics as nm
    ref = mpi_ref.allreduce(xs, "sum", "bfloat16")[0]
    for g in got:
        assert np.array_equal(nm.to_f64(g, "bfloat16"), ref)


@pytest.mark.parametrize("R", [2, 4, 8])
def test_nvls_reducescatter_and_allgather(R):
    n = 30011
    xs = synth.inputs(R, R * n, "float32", "uniform")
    algo = P.nvls_reducescatter(R, 2)
    want = sim.simulate(irparse.parse(algo.to_xml()), xs, n, "float32", "sum")
    got = _run(algo, xs, n, "float32", "sum", out_elems=n)
    for g, w in zip(got, want):
        assert np.array_equal(g.view(np.uint32), w.view(np.uint32))
    xs = synth.inputs(R, n, "int32", "pattern")
    got = _run(P.nvls_allgather(R, 2), xs, n, "int32", out_elems=R * n)
    for g, w in zip(got, mpi_ref.allgather(xs)):
        assert np.array_equal(g, w)


def test_nvls_prod_rejected():
    import gpu_util
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    R, n = 4, 1000
    xs = synth.inputs(R, n, "float32", "uniform")
    with pytest.raises(runtime.MscclError) as ei:
        gpu_util.run_program(P.nvls_allreduce(R).to_xml(), xs, n, "float32", "prod")
    assert ei.value.code == 4


def test_multicast_hardware_path():
    """The hardware form of the multimem ops: NVLS buffers bound to an NVSwitch multicast
    object (mscclNvlsAlloc) and multimem.ld_reduce / multimem.st on the multicast address.
    Every visible GPU joins (one rank per GPU); on a one-GPU box the team has one member, so
    the reduction is the identity, but the multicast object, its mappings and the multimem
    instructions all run on the hardware. Outputs are checked against the oracle and the
    device counter proves the multicast path executed."""
    import torch
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    ndev = torch.cuda.device_count()
    if not all(runtime.nvls_supported(d) for d in range(ndev)):
        pytest.skip("CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED is 0 on this box")
    R = ndev
    comms = runtime.Comm.init_all(list(range(R)))
    try:
        n = 65536 * R
        nbytes = 2 * n * 4 * 2   # in + out, fp32, headroom
        try:
            bufs, ptrs = runtime.nvls_alloc(comms, nbytes)
        except runtime.MscclError as e:   # e.g. cuMulticastCreate refused (profiles/r02/mcprobe.txt)
            pytest.skip("NVSwitch multicast object unavailable on this box: %s" % e)
        try:
            for dtype, tdt, build, out_mul in (("float32", torch.float32, P.nvls_allreduce, 1),
                                               ("bfloat16", torch.bfloat16, P.nvls_allreduce, 1),
                                               ("int32", torch.int32, P.nvls_allgather, R)):
                w = torch.tensor([], dtype=tdt).element_size()
                count = n // R if out_mul == R else n
                xs = synth.inputs(R, count, dtype, "uniform" if dtype != "int32" else "pattern")
                algo = build(R, 2)
                want = sim.simulate(irparse.parse(algo.to_xml()), xs, count, dtype, "sum")
                progs = [c.load(algo.to_xml()) for c in comms]
                send, recv = [], []
                for q in range(R):
                    b = bufs[q]
                    s = b[:count * w].view(tdt)
                    r = b[count * w + 4096 - (count * w) % 4096:][:count * out_mul * w].view(tdt)
                    s.copy_(torch.from_numpy(xs[q].view(np.uint8).copy()).cuda(q).view(tdt))
                    send.append(s)
                    recv.append(r)
                before = [c.stats()["multicast_pieces"] for c in comms]
                with runtime.group():
                    for c, p_, s, r in zip(comms, progs, send, recv):
                        c.run(p_, s, r, count)
                torch.cuda.synchronize()
                for q in range(R):
                    got = recv[q].cpu().view(torch.uint8).numpy()
                    assert np.array_equal(got, np.ascontiguousarray(want[q]).view(np.uint8)), (dtype, q)
                    assert comms[q].stats()["multicast_pieces"] > before[q], dtype
                for c, p_ in zip(comms, progs):
                    c.unload(p_)
        finally:
            runtime.nvls_free(comms, ptrs)
    finally:
        for c in comms:
            c.destroy()


@pytest.mark.parametrize("R", [2, 4, 8])
@pytest.mark.parametrize("dtype", ["bfloat16", "float32", "int32"])
def test_mixed_ring_rs_multimem_ag_bit_exact(R, dtype):
    """Connection ops and multimem ops in one program (the multimem kernel variant runs the
    ring part too): bit-exact with the oracle."""
    n = 50021
    xs = synth.inputs(R, n, dtype, "uniform" if dtype != "int32" else "int")
    algo = P.ring_rs_multimem_ag_allreduce(R, 2)
    want = sim.simulate(irparse.parse(algo.to_xml()), xs, n, dtype, "sum")
    got = _run(algo, xs, n, dtype, "sum")
    for g, w in zip(got, want):
        assert np.array_equal(np.asarray(g).view(np.uint8), np.asarray(w).view(np.uint8))
