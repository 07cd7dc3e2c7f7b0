"""Pins for the oracle IR simulator (oracle/sim.py) — none of them re-derives its code.

* brute force: on integer-valued inputs every reduction order is exact, so the simulator
  must equal the MPI definitions (oracle/mpi_ref.py) bit for bit;
* the ring closed form: chunk c = x_c (+) (x_{c-1} (+) (... (+) (x_{c+2} (+)
  x_{c+1}))), computed here with torch's own bf16/fp16/fp32 arithmetic;
* all-pairs / one-shot = ascending fold ((x_0 (+) x_1) (+) x_2) ... (reading R7);
* invariances: bits do not depend on tile size, FIFO slots, instances or in-place form;
* deadlock fixtures of §4.2 / P:L1317-1319.
"""
import numpy as np
import pytest
import torch

import synth
from oracle import irparse, mpi_ref, sim
from oracle import numerics as nm
from paper_conf_asplos_cowanmmsx23_b200 import programs as P

TORCH = {"bfloat16": torch.bfloat16, "float16": torch.float16, "float32": torch.float32}


def _parse(algo):
    return irparse.parse(algo.to_xml())


def _t(x, dtype):
    if dtype == "bfloat16":
        return torch.from_numpy(x.view(np.int16).copy()).view(torch.bfloat16)
    return torch.from_numpy(x.copy())


def _np(t, dtype):
    if dtype == "bfloat16":
        return t.view(torch.int16).numpy().view(np.uint16)
    return t.numpy()


def _exact_inputs(R, n, dtype, op, seed=7):
    xs = synth.inputs(R, n, dtype, "intval" if dtype in nm.FLOATS else "int", seed=seed)
    if op == "prod":  # keep every partial product exact: values in {+-1, +-2}
        g = np.random.default_rng(seed)
        xs = [nm.from_f64(g.choice([-2.0, -1.0, 1.0, 2.0], n), dtype) for _ in range(R)]
    return xs


def _eq(a, b):
    return np.array_equal(np.asarray(a).view(np.uint8), np.asarray(b).view(np.uint8))


PROGS_AR = [
    ("ring", lambda R: P.ring_allreduce(R)),
    ("ring_inplace", lambda R: P.ring_allreduce(R, inplace=True)),
    ("ring_channels", lambda R: P.ring_allreduce(R, channels=R, instances=2)),
    ("ring_split", lambda R: P.ring_allreduce(R, channels=R, split_phases=True)),
    ("ring_k2", lambda R: P.ring_allreduce(R, rings=2)),
    ("allpairs", lambda R: P.allpairs_allreduce(R)),
    ("oneshot", lambda R: P.oneshot_allreduce(R)),
]


@pytest.mark.parametrize("R", [2, 4, 8])
@pytest.mark.parametrize("name,build", PROGS_AR)
@pytest.mark.parametrize("dtype,op", [("float32", "sum"), ("bfloat16", "sum"), ("float16", "max"),
                                      ("int32", "sum"), ("float32", "prod"), ("int32", "min")])
def test_allreduce_programs_equal_brute_force(R, name, build, dtype, op):
    n = 1000 + 3 * R  # ragged: not a multiple of the chunk count or the vector width
    algo = _parse(build(R))
    xs = _exact_inputs(R, n, dtype, op)
    out = sim.simulate(algo, xs, n, dtype, op)
    ref = mpi_ref.allreduce(xs, op, dtype)
    for o, r in zip(out, ref):
        assert _eq(o, nm.from_f64(r, dtype) if dtype in nm.FLOATS else r)


@pytest.mark.parametrize("N,G", [(2, 2), (2, 3), (2, 4), (4, 2)])
def test_hierarchical_equals_brute_force(N, G):
    R = N * G
    algo = _parse(P.hierarchical_allreduce(N, G))
    n = 777
    xs = _exact_inputs(R, n, "float32", "sum")
    out = sim.simulate(algo, xs, n, "float32", "sum")
    ref = mpi_ref.allreduce(xs, "sum", "float32")
    assert all(_eq(o, r.astype(np.float32)) for o, r in zip(out, ref))


@pytest.mark.parametrize("R", [2, 4, 8])
@pytest.mark.parametrize("r", [1, 2, 4])
def test_allgather_reducescatter_equal_brute_force(R, r):
    n = 333
    xs = synth.inputs(R, n, "int32", "pattern")
    out = sim.simulate(_parse(P.ring_allgather(R, 2, r)), xs, n, "int32")
    assert all(_eq(o, e) for o, e in zip(out, mpi_ref.allgather(xs)))
    out = sim.simulate(_parse(P.allpairs_allgather(R, r)), xs, n, "int32")
    assert all(_eq(o, e) for o, e in zip(out, mpi_ref.allgather(xs)))
    xs = _exact_inputs(R, R * n, "bfloat16", "sum")
    out = sim.simulate(_parse(P.ring_reducescatter(R, 2, r)), xs, n, "bfloat16", "sum")
    ref = mpi_ref.reducescatter(xs, n, "sum", "bfloat16")
    assert all(_eq(o, nm.from_f64(e, "bfloat16")) for o, e in zip(out, ref))


@pytest.mark.parametrize("N,G", [(1, 2), (1, 4), (1, 8), (2, 2), (2, 4), (4, 2)])
@pytest.mark.parametrize("r", [1, 2])
@pytest.mark.parametrize("dtype", ["int32", "bfloat16", "float64"])
def test_alltoall_equals_transpose(N, G, r, dtype):
    R = N * G
    n = 129
    xs = synth.inputs(R, R * n, dtype, "pattern")
    out = sim.simulate(_parse(P.alltoall_twostep(N, G, r)), xs, n, dtype)
    assert all(_eq(o, e) for o, e in zip(out, mpi_ref.alltoall(xs, n)))


@pytest.mark.parametrize("N,G", [(1, 4), (2, 3), (3, 2)])
def test_alltonext_definition(N, G):
    R = N * G
    n = 250
    xs = synth.inputs(R, n, "int32", "pattern")
    out = sim.simulate(_parse(P.alltonext(N, G)), xs, n, "int32")
    ref = mpi_ref.alltonext(xs)
    for q in range(1, R):
        assert _eq(out[q], ref[q])


def _ring_closed_form(xs, dtype, E, K=1):
    """chunk c = x_c + (x_{c-1} + (... + (x_{c+2} + x_{c+1}))) per element;
    with K logical rings over K*R chunks, chunk c starts on rank (c mod R) + 1 (Fig. 3b with
    offset (c div R)*R)."""
    R = len(xs)
    ts = [_t(x, dtype) for x in xs]
    n = ts[0].numel()
    out = torch.empty_like(ts[0])
    for c in range(K * R):
        lo, hi = c * E, min((c + 1) * E, n)
        if lo >= hi:
            continue
        acc = ts[(c + 1) % R][lo:hi]
        for k in range(2, R + 1):
            acc = ts[(c + k) % R][lo:hi] + acc
        out[lo:hi] = acc
    return _np(out, dtype)


@pytest.mark.parametrize("R", [2, 4, 8])
@pytest.mark.parametrize("dtype", ["bfloat16", "float16", "float32"])
def test_ring_matches_closed_form_bitwise(R, dtype):
    n = 4096 + 40
    xs = synth.inputs(R, n, dtype, "uniform")
    V = 16 // nm.elem_bytes(dtype)
    E = -(-(-(-n // R)) // V) * V
    want = _ring_closed_form(xs, dtype, E)
    for algo in (P.ring_allreduce(R), P.ring_allreduce(R, inplace=True),
                 P.ring_allreduce(R, channels=R, split_phases=True)):  # R26: same chunk paths
        out = sim.simulate(_parse(algo), xs, n, dtype, "sum")
        for o in out:
            assert _eq(o, want)


@pytest.mark.parametrize("R", [2, 4, 8])
@pytest.mark.parametrize("K", [2, 3])
def test_k_rings_match_closed_form_bitwise(R, K):
    """R27: K logical rings over K*R chunks; chunk geometry per reading R1 with K*R chunks."""
    n = 4096 + 40
    dtype = "bfloat16"
    xs = synth.inputs(R, n, dtype, "uniform")
    V = 16 // nm.elem_bytes(dtype)
    E = -(-(-(-n // (K * R))) // V) * V
    want = _ring_closed_form(xs, dtype, E, K)
    for algo in (P.ring_allreduce(R, rings=K), P.ring_allreduce(R, rings=K, inplace=True)):
        out = sim.simulate(_parse(algo), xs, n, dtype, "sum", slots=8)
        for o in out:
            assert _eq(o, want)


@pytest.mark.parametrize("R", [2, 4, 8])
@pytest.mark.parametrize("dtype", ["bfloat16", "float16"])
def test_allpairs_and_oneshot_equal_ascending_fold(R, dtype):
    n = 2048 + 24
    xs = synth.inputs(R, n, dtype, "uniform")
    ts = [_t(x, dtype) for x in xs]
    acc = ts[0]
    for t in ts[1:]:
        acc = acc + t
    want = _np(acc, dtype)
    for algo in (P.allpairs_allreduce(R), P.oneshot_allreduce(R), P.allpairs_allreduce(R, instances=2)):
        for o in sim.simulate(_parse(algo), xs, n, dtype, "sum"):
            assert _eq(o, want)


def test_tiling_slots_instances_do_not_change_bits():
    R, n, dtype = 8, 8192, "bfloat16"
    xs = synth.inputs(R, n, dtype, "uniform")
    base = sim.simulate(_parse(P.ring_allreduce(R)), xs, n, dtype)
    for slot_bytes in (64, 256, 1000, 4096):
        for slots in (2, 3, 8):
            out = sim.simulate(_parse(P.ring_allreduce(R)), xs, n, dtype, slots=slots, slot_bytes=slot_bytes)
            assert all(_eq(a, b) for a, b in zip(base, out))
    for r in (2, 4):   # E divisible by r: every sub-chunk follows its parent's ring path (reading R5)
        out = sim.simulate(_parse(P.ring_allreduce(R, instances=r)), xs, n, dtype)
        assert all(_eq(a, b) for a, b in zip(base, out))
    out = sim.simulate(_parse(P.ring_allreduce(R, channels=R)), xs, n, dtype)
    assert all(_eq(a, b) for a, b in zip(base, out))


def test_count_zero_and_tiny_counts():
    algo = _parse(P.ring_allreduce(4))
    xs = [np.zeros(0, np.float32) for _ in range(4)]
    assert all(o.size == 0 for o in sim.simulate(algo, xs, 0, "float32"))
    for n in (1, 3, 5, 17):   # most chunks empty
        xs = _exact_inputs(4, n, "float32", "sum")
        out = sim.simulate(algo, xs, n, "float32")
        ref = mpi_ref.allreduce(xs, "sum", "float32")
        assert all(_eq(o, r.astype(np.float32)) for o, r in zip(out, ref))


def test_scratch_tail_garbage_never_reaches_output():
    # all-pairs receives ragged chunks into full-size scratch chunks (reading R2)
    R, n = 4, 13
    xs = _exact_inputs(R, n, "float32", "sum")
    out = sim.simulate(_parse(P.allpairs_allreduce(R)), xs, n, "float32")
    ref = mpi_ref.allreduce(xs, "sum", "float32")
    assert all(_eq(o, r.astype(np.float32)) for o, r in zip(out, ref))


ONE_RANK = [
    ("ring", lambda: P.ring_allreduce(1), "allreduce"),
    ("ring_inplace", lambda: P.ring_allreduce(1, inplace=True), "allreduce"),
    ("ring_instances", lambda: P.ring_allreduce(1, instances=2), "allreduce"),
    ("ring_k2", lambda: P.ring_allreduce(1, rings=2), "allreduce"),
    ("allpairs", lambda: P.allpairs_allreduce(1), "allreduce"),
    ("oneshot", lambda: P.oneshot_allreduce(1), "allreduce"),
    ("allgather", lambda: P.ring_allgather(1, 2, 2), "allgather"),
    ("reducescatter", lambda: P.ring_reducescatter(1, 2, 2), "reducescatter"),
    ("alltoall", lambda: P.alltoall_twostep(1, 1), "alltoall"),
    ("nvls", lambda: P.nvls_allreduce(1), "allreduce"),
]


@pytest.mark.parametrize("name,build,coll", ONE_RANK, ids=[x[0] for x in ONE_RANK])
def test_one_rank_programs_copy_their_input(name, build, coll):
    """Degenerate case R = 1: every collective's output is the input (the MPI definitions with
    one rank); the ring builders used to leave the output unwritten (DSL refused the ring
    AllReduce, the ReduceScatter was empty)."""
    algo = _parse(build())
    n = 1000
    xs = synth.inputs(1, n, "int32", "int")
    out = sim.simulate(algo, xs, n, "int32", "sum")
    assert np.array_equal(out[0][:n], xs[0][:n])
