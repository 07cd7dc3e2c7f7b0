"""GPU parity: the CUDA interpreter (through the C ABI) vs the CPU oracle, element by element.

Gate G1: bit-exact with the oracle simulator executing the same IR for every
dtype (one rounding per reduce instruction in both); AllGather/AllToAll/int also
bit-exact with the brute-force definitions. Gate G2: float results within the stated
tolerance of the fp64 definition (fp32 per-element normwise <= 1e-6, fp16 <= 1e-2,
bf16 l2-relative <= 1e-2; north_star / DESIGN.md "Tolerances").

All ranks are virtual ranks on cuda:0 (one cooperative launch). A small FIFO slot
(16 KiB) makes the pipelining loop run several tiles even at test sizes.
"""
import numpy as np
import pytest

import synth
from oracle import irparse, mpi_ref, sim
from oracle import numerics as nm
from paper_conf_asplos_cowanmmsx23_b200 import programs as P

pytestmark = pytest.mark.gpu

SLOT = 16384


@pytest.fixture(scope="module", autouse=True)
def small_slots():
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    runtime.set_param("MSCCL_SLOT_BYTES", SLOT)
    runtime.set_param("MSCCL_LL_SLOT_BYTES", SLOT)
    runtime.set_param("MSCCL_LL128_SLOT_BYTES", SLOT)
    runtime.set_param("MSCCL_SLOTS", 4)
    runtime.set_param("MSCCL_TIMEOUT_S", 5)
    yield


def _gpu():
    import gpu_util
    return gpu_util


def _bits_equal(a, b):
    return np.array_equal(np.asarray(a).view(np.uint8), np.asarray(b).view(np.uint8))


def _g2(out, xs, op, dtype):
    if dtype not in nm.FLOATS or op != "sum":
        return
    ref = mpi_ref.allreduce(xs, op, dtype)[0]
    got = nm.to_f64(out, dtype)
    err = np.abs(got - ref)
    if dtype == "bfloat16":
        assert np.linalg.norm(err) <= 1e-2 * np.linalg.norm(ref)
    else:
        scale = np.sum([np.abs(nm.to_f64(x, dtype)) for x in xs], axis=0)
        tol = 1e-6 if dtype == "float32" else 1e-2
        assert np.all(err <= tol * scale + 1e-300)


def _check_allreduce(ir_text, R, n, dtype, op, dist="uniform"):
    xs = synth.inputs(R, n, dtype, dist if dtype in nm.FLOATS else "int")
    algo = irparse.parse(ir_text)
    want = sim.simulate(algo, xs, n, dtype, op)
    got = _gpu().run_program(ir_text, xs, n, dtype, op)
    for q in range(R):
        assert _bits_equal(got[q], want[q]), "rank %d differs from the oracle" % q
    _g2(got[0], xs, op, dtype)


AR = [
    ("ring", lambda R: P.ring_allreduce(R)),
    ("ring_inplace", lambda R: P.ring_allreduce(R, inplace=True)),
    ("ring_channels_instances", lambda R: P.ring_allreduce(R, channels=R, instances=2)),
    ("ring_split", lambda R: P.ring_allreduce(R, channels=R, split_phases=True)),
    ("ring_k2", lambda R: P.ring_allreduce(R, rings=2)),
    ("ring_LL", lambda R: P.ring_allreduce(R, protocol="LL")),
    ("ring_LL128", lambda R: P.ring_allreduce(R, instances=2, protocol="LL128")),
    ("allpairs_LL128", lambda R: P.allpairs_allreduce(R, protocol="LL128")),
    ("allpairs_LL", lambda R: P.allpairs_allreduce(R)),
    ("allpairs_simple", lambda R: P.allpairs_allreduce(R, protocol="Simple")),
    ("oneshot_LL", lambda R: P.oneshot_allreduce(R)),
]


@pytest.mark.parametrize("R", [2, 4, 8])
@pytest.mark.parametrize("name,build", AR, ids=[a[0] for a in AR])
@pytest.mark.parametrize("dtype,op", [("bfloat16", "sum"), ("float16", "sum"), ("float32", "sum"),
                                      ("int32", "sum"), ("float32", "max"), ("bfloat16", "min")])
def test_allreduce_bit_exact_vs_oracle(R, name, build, dtype, op):
    n = 3 * 8192 * R + 37          # several tiles per chunk + a ragged tail
    _check_allreduce(build(R).to_xml(), R, n, dtype, op)


@pytest.mark.parametrize("dtype,op", [("float64", "sum"), ("int8", "sum"), ("uint8", "max"), ("int64", "prod"),
                                      ("uint32", "sum"), ("uint64", "min"), ("float16", "prod")])
def test_allreduce_other_types(dtype, op):
    _check_allreduce(P.ring_allreduce(4).to_xml(), 4, 20011, dtype, op)


@pytest.mark.parametrize("N,G", [(2, 2), (2, 3), (2, 4), (4, 2)])
def test_hierarchical(N, G):
    _check_allreduce(P.hierarchical_allreduce(N, G).to_xml(), N * G, 50000, "bfloat16", "sum")


@pytest.mark.parametrize("n", [1, 2, 7, 8, 9, 63, 4096, 4097])
def test_tiny_and_ragged_counts(n):
    _check_allreduce(P.ring_allreduce(8).to_xml(), 8, n, "bfloat16", "sum")
    _check_allreduce(P.allpairs_allreduce(8).to_xml(), 8, n, "float32", "sum")


@pytest.mark.parametrize("R", [2, 4, 8])
@pytest.mark.parametrize("r", [1, 2, 4])
def test_allgather_reducescatter(R, r):
    n = 5000 + 3
    xs = synth.inputs(R, n, "int32", "pattern")
    got = _gpu().run_program(P.ring_allgather(R, 2, r).to_xml(), xs, n, "int32", out_elems=R * n)
    for g, e in zip(got, mpi_ref.allgather(xs)):
        assert _bits_equal(g, e)
    if R * 2 * (R - 1) * r <= 296:  # all-pairs: 2(R-1) thread blocks per rank and instance, co-resident
        got = _gpu().run_program(P.allpairs_allgather(R, r).to_xml(), xs, n, "int32", out_elems=R * n)
        for g, e in zip(got, mpi_ref.allgather(xs)):
            assert _bits_equal(g, e)
    xs = synth.inputs(R, R * n, "bfloat16", "uniform")
    ir = P.ring_reducescatter(R, 2, r).to_xml()
    want = sim.simulate(irparse.parse(ir), xs, n, "bfloat16", "sum")
    got = _gpu().run_program(ir, xs, n, "bfloat16", "sum", out_elems=n)
    for g, w in zip(got, want):
        assert _bits_equal(g, w)


@pytest.mark.parametrize("N,G", [(1, 2), (1, 4), (1, 8), (2, 4), (4, 2)])
@pytest.mark.parametrize("dtype", ["int32", "bfloat16", "float64", "int8"])
def test_alltoall(N, G, dtype):
    R = N * G
    n = 3001
    xs = synth.inputs(R, R * n, dtype, "pattern")
    got = _gpu().run_program(P.alltoall_twostep(N, G).to_xml(), xs, n, dtype, out_elems=R * n)
    for g, e in zip(got, mpi_ref.alltoall(xs, n)):
        assert _bits_equal(g, e)


def test_alltonext():
    R, n = 6, 7777
    xs = synth.inputs(R, n, "int32", "pattern")
    got = _gpu().run_program(P.alltonext(2, 3).to_xml(), xs, n, "int32")
    ref = mpi_ref.alltonext(xs)
    for q in range(1, R):
        assert _bits_equal(got[q], ref[q])


def test_repeated_launches_keep_counters_consistent():
    """Connection counters and semaphores persist across launches (reading R4)."""
    R, n = 8, 100000
    ir = P.allpairs_allreduce(R, protocol="Simple").to_xml()
    xs = synth.inputs(R, n, "float32", "uniform")
    want = sim.simulate(irparse.parse(ir), xs, n, "float32")
    for _ in range(3):
        got = _gpu().run_program(ir, xs, n, "float32")
        assert all(_bits_equal(g, w) for g, w in zip(got, want))


@pytest.mark.parametrize("slots", [2, 3, 5, 8])
@pytest.mark.parametrize("proto", ["Simple", "LL", "LL128"])
def test_slot_counts(slots, proto):
    """FIFO slot index of message k is k mod s (§6.1): power-of-two slot counts
    take a mask, others the remainder; every protocol, many tiles (wrap-around many times)."""
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    runtime.set_param("MSCCL_SLOTS", slots)
    try:
        n = 3 * 8192 * 4 + 37
        _check_allreduce(P.ring_allreduce(4, protocol=proto).to_xml(), 4, n, "bfloat16", "sum")
        if slots >= 3:  # two interleaved rings need s >= 3 (reading R27, V9)
            _check_allreduce(P.ring_allreduce(4, instances=2, rings=2, protocol=proto).to_xml(), 4, n, "float32",
                             "sum")
    finally:
        runtime.set_param("MSCCL_SLOTS", 4)


@pytest.mark.parametrize("name", ["ring", "ring_inplace", "allpairs", "oneshot", "allgather", "reducescatter",
                                  "alltoall", "nvls"])
def test_one_rank_programs(name):
    """Degenerate case R = 1 on a one-rank communicator: output = input, bit for bit."""
    build = {"ring": lambda: P.ring_allreduce(1), "ring_inplace": lambda: P.ring_allreduce(1, inplace=True),
             "allpairs": lambda: P.allpairs_allreduce(1, protocol="Simple"), "oneshot": lambda: P.oneshot_allreduce(1),
             "allgather": lambda: P.ring_allgather(1, 2, 2), "reducescatter": lambda: P.ring_reducescatter(1, 2, 2),
             "alltoall": lambda: P.alltoall_twostep(1, 1), "nvls": lambda: P.nvls_allreduce(1)}[name]
    n = 4099
    xs = synth.inputs(1, n, "float32", "uniform")
    got = _gpu().run_program(build().to_xml(), xs, n, "float32", "sum")
    assert _bits_equal(got[0][:n], xs[0][:n])


@pytest.mark.gpu
@pytest.mark.parametrize("hints", [25, 9])
@pytest.mark.parametrize("name", ["ring_allreduce", "ring_reducescatter"])
def test_pulled_first_hops_bit_exact(name, hints):
    """Reading R30: the ring's first hops read the sender's input chunk (MSCCL_DIRECT_HINTS
    bit 4, the default) or go through the FIFO (9); both bit-exact with the oracle at a ragged
    count over several tiles, bf16 and int32."""
    import gpu_util
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    old = runtime.get_param("MSCCL_DIRECT_HINTS"), runtime.get_param("MSCCL_SLOT_BYTES")
    runtime.set_param("MSCCL_DIRECT_HINTS", hints)
    runtime.set_param("MSCCL_SLOT_BYTES", 8192)
    try:
        R = 8
        algo = P.ring_allreduce(R, instances=2) if name == "ring_allreduce" else P.ring_reducescatter(R, 1, 2)
        text = algo.to_xml()
        for dtype in ("bfloat16", "int32"):
            cnt = R * 2 * 3001 + 5 if name == "ring_allreduce" else 2 * 3001 + 5   # ragged chunks (R1)
            n_in = cnt if name == "ring_allreduce" else R * cnt
            xs = synth.inputs(R, n_in, dtype, "int" if dtype == "int32" else "uniform", seed=hints)
            want = sim.simulate(irparse.parse(text), xs, cnt, dtype, "sum")
            got = gpu_util.run_program(text, xs, cnt, dtype, "sum", out_elems=cnt)
            for r in range(R):
                assert np.array_equal(got[r][:cnt].view(np.uint8), want[r][:cnt].view(np.uint8)), (name, hints, dtype, r)
    finally:
        runtime.set_param("MSCCL_DIRECT_HINTS", old[0])
        runtime.set_param("MSCCL_SLOT_BYTES", old[1])
