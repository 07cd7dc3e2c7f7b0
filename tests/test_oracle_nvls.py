"""Pins for the multimem (NVLS) ops of the oracle (reading R23).

* numerics.mreduce against exact rational arithmetic: a 16-bit float sum accumulates in fp32
  and rounds once (1 + 2^-8 + 2^-8 in bf16 is 1 + 2^-7, where chained bf16 adds give 1);
  integers wrap; max/min are exact; prod is rejected;
* the NVLS programs (mrs AllReduce, mrd ReduceScatter, mst AllGather) at R in {2,4,8} x
  instances in {1,2,4}: the simulator's outputs equal the brute-force MPI definition exactly
  on integer-valued inputs and equal an independently rounded exact rational sum on random
  bf16 inputs; the symbolic postcondition holds with rank-identical trees; the validator and
  the race detector accept them;
* negative pins: multimem ops on scratch and mismatched multimem thread blocks (V11), two
  ranks storing to one chunk (a race), and the DSL refusing to read a multimem result or to
  reduce a modified input.
"""
from fractions import Fraction

import numpy as np
import pytest

import synth
from oracle import irparse, mpi_ref, races, sim, symbolic, validate
from oracle import numerics as nm
from paper_conf_asplos_cowanmmsx23_b200 import dsl
from paper_conf_asplos_cowanmmsx23_b200 import programs as P


def _bf16_value(bits):
    u = int(bits) << 16
    sign = -1 if u >> 31 else 1
    e = (u >> 23) & 0xFF
    m = u & 0x7FFFFF
    if e == 0:
        return sign * Fraction(m, 1 << 23) * Fraction(1, 1 << 126)
    return sign * (1 + Fraction(m, 1 << 23)) * (Fraction(2) ** (e - 127))


def _round_bf16(x):
    """Independent RNE rounding of a rational to bf16 (8 significant bits), normal range."""
    if x == 0:
        return 0
    sign = -1 if x < 0 else 1
    a = abs(x)
    e = 0
    while a >= 2:
        a /= 2
        e += 1
    while a < 1:
        a *= 2
        e -= 1
    scaled = a * 128                      # 1.xxxxxxx -> 8 significant bits
    fl = scaled.numerator // scaled.denominator
    rem = scaled - fl
    if rem > Fraction(1, 2) or (rem == Fraction(1, 2) and fl % 2 == 1):
        fl += 1
    return sign * Fraction(fl, 128) * Fraction(2) ** e


def _bits_of(x):
    return int(nm.f32_to_bf16(np.array([float(x)], dtype=np.float64).astype(np.float32))[0])


def test_mreduce_single_rounding_bf16():
    one, tiny = _bits_of(1.0), _bits_of(2.0 ** -8)
    vals = [np.array([one], np.uint16), np.array([tiny], np.uint16), np.array([tiny], np.uint16)]
    got = nm.mreduce(vals, "sum", "bfloat16")
    assert _bf16_value(got[0]) == 1 + Fraction(1, 128)
    chained = nm.reduce(nm.reduce(vals[0], vals[1], "sum", "bfloat16"), vals[2], "sum", "bfloat16")
    assert _bf16_value(chained[0]) == 1   # one rounding per instruction (reading R6) differs


def test_mreduce_matches_exact_rational_rounding():
    rng = np.random.default_rng(7)
    for R in (2, 4, 8):
        xs = [synth.rank_input(q, 4000, "bfloat16", "uniform") for q in range(R)]
        got = nm.mreduce(xs, "sum", "bfloat16")
        checked = 0
        for e in rng.integers(0, 4000, 300):
            vals = [_bf16_value(x[e]) for x in xs]
            partial, exact_acc = vals[0], True
            for v in vals[1:]:                       # fp32 accumulation exact at every step?
                partial += v
                f = Fraction(float(np.float32(float(partial))))
                exact_acc = exact_acc and f == partial
            if not exact_acc or partial == 0:
                continue
            assert _bf16_value(got[e]) == _round_bf16(partial), (R, e)
            checked += 1
        assert checked > 200


def test_mreduce_ints_wrap_and_minmax_exact():
    a = np.array([2 ** 31 - 1, -5], np.int32)
    b = np.array([1, 3], np.int32)
    assert list(nm.mreduce([a, b], "sum", "int32")) == [-2 ** 31, -2]
    xs = [synth.rank_input(q, 1000, "float32", "uniform") for q in range(8)]
    assert np.array_equal(nm.mreduce(xs, "max", "float32"), np.max(np.stack(xs), axis=0))
    assert np.array_equal(nm.mreduce(xs, "min", "float32"), np.min(np.stack(xs), axis=0))
    with pytest.raises(ValueError):
        nm.mreduce(xs, "prod", "float32")


def _al(a):
    return irparse.parse(a.to_xml())


@pytest.mark.parametrize("R", [2, 4, 8])
@pytest.mark.parametrize("r", [1, 2, 4])
def test_nvls_programs_exact_on_integer_inputs(R, r):
    n = 37 * R * r + 5
    for dtype in ("bfloat16", "float32", "int32"):
        dist = "intval" if dtype != "int32" else "int"
        xs = synth.inputs(R, n, dtype, dist)
        al = _al(P.nvls_allreduce(R, r))
        got = sim.simulate(al, xs, n, dtype, "sum")
        want = mpi_ref.allreduce(xs, "sum", dtype)
        for g, w in zip(got, want):
            assert np.array_equal(nm.to_f64(g, dtype), np.asarray(w, dtype=np.float64)), dtype
    xs = synth.inputs(R, R * n, "int32", "int")
    got = sim.simulate(_al(P.nvls_reducescatter(R, r)), xs, n, "int32", "sum")
    for q in range(R):
        want = np.sum(np.stack([x[q * n:(q + 1) * n].astype(np.int64) for x in xs]), axis=0)
        assert np.array_equal(got[q].astype(np.int64), (want + 2 ** 31) % 2 ** 32 - 2 ** 31)
    xs = synth.inputs(R, n, "bfloat16", "pattern")
    got = sim.simulate(_al(P.nvls_allgather(R, r)), xs, n, "bfloat16")
    for g, w in zip(got, mpi_ref.allgather(xs)):
        assert np.array_equal(g, w)


@pytest.mark.parametrize("R", [2, 4, 8])
def test_nvls_allreduce_float_closed_form(R):
    """bf16 random inputs: every output element is the bf16 rounding of the exact sum when
    the fp32 accumulation is exact (independent rational arithmetic)."""
    n = 2000
    xs = synth.inputs(R, n, "bfloat16", "uniform")
    got = sim.simulate(_al(P.nvls_allreduce(R, 2)), xs, n, "bfloat16", "sum")
    rng = np.random.default_rng(3)
    checked = 0
    for e in rng.integers(0, n, 200):
        vals = [_bf16_value(x[e]) for x in xs]
        s = sum(vals[1:], vals[0])
        ok = all(Fraction(float(np.float32(float(sum(vals[1:k + 1], vals[0]))))) == sum(vals[1:k + 1], vals[0])
                 for k in range(1, R))
        if not ok or s == 0:
            continue
        for q in range(R):
            assert _bf16_value(got[q][e]) == _round_bf16(s)
        checked += 1
    assert checked > 100


@pytest.mark.parametrize("R", [2, 4, 8])
@pytest.mark.parametrize("build", [P.nvls_allreduce, P.nvls_reducescatter, P.nvls_allgather])
def test_nvls_symbolic_validator_races(R, build):
    for r in (1, 2, 4):
        al = _al(build(R, r))
        validate.validate(al, nranks=R, races=True)
        symbolic.check(al)
        assert races.find_races(al) == []


def test_v11_multimem_scratch_and_block_mismatch():
    a = P.nvls_allreduce(4)
    bad = a.to_xml().replace('type="mrs" srcbuf="i"', 'type="mrs" srcbuf="s"', 1).replace(
        's_chunks="0"', 's_chunks="4"')
    with pytest.raises(validate.ValidationError, match="^V11"):
        validate.validate(irparse.parse(bad), nranks=4)
    al = _al(P.nvls_allreduce(4))
    g = al.gpus[1]
    g.tbs.insert(0, irparse.TB(id=0, send=-1, recv=-1, chan=5,
                               steps=[irparse.Step(0, "nop", "-", -1, "-", -1, 1, [], False)]))
    g.tbs[1].id = 1
    with pytest.raises(validate.ValidationError, match="^V11"):
        validate.validate(al, nranks=4)


def test_two_ranks_storing_one_chunk_race():
    al = _al(P.nvls_allgather(4))
    st = al.gpus[2].tbs[0].steps[0]
    st.dstoff = 1           # rank 2 now also stores into block 1 (rank 1's)
    rs = races.find_races(al)
    assert rs and any(r.loc[1] == "o" and r.loc[2] == 1 for r in rs)


def test_dsl_multimem_rules():
    with pytest.raises(dsl.DSLError, match="final"):
        with dsl.Program("x", dsl.AllReduce(2, 2)):
            dsl.chunk(0, "in", 0).multimem_reduce("out", 0)
            dsl.chunk(1, "out", 0)
    with pytest.raises(dsl.DSLError, match="unmodified"):
        with dsl.Program("y", dsl.AllReduce(2, 2, inplace=True)):
            c = dsl.chunk(1, "in", 0).copy(0, "in", 0)
            dsl.chunk(0, "in", 0).multimem_reduce("out", 0)


def test_sampled_oracle_evaluates_multimem_nodes():
    """oracle/sampled.py (used at bench sizes) agrees with the full simulation of the NVLS
    AllReduce bit for bit, including the single rounding of the multimem fold."""
    from oracle import sampled
    R, n = 8, 5000
    xs = synth.inputs(R, n, "bfloat16", "uniform")
    al = _al(P.nvls_allreduce(R, 2))
    full = sim.simulate(al, xs, n, "bfloat16", "sum")
    idx = np.arange(0, n, 7)
    for q in (0, 5):
        got = sampled.allreduce_at(al, lambda r, i: xs[r][i], n, "bfloat16", "sum", idx, rank=q)
        assert np.array_equal(got, full[q][idx])


@pytest.mark.parametrize("R", [2, 4, 8])
def test_mixed_ring_rs_multimem_ag(R):
    """A program mixing connection ops and multimem ops (ring ReduceScatter + multimem
    AllGather): postcondition, rank-identical trees, race free (with the loader's direct
    marking), brute-force exact on integer-valued inputs."""
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    for r in (1, 2):
        algo = P.ring_rs_multimem_ag_allreduce(R, r)
        ir = algo.to_xml()
        al = irparse.parse(ir)
        validate.validate(al, nranks=R, races=True)
        symbolic.check(al)
        assert races.check_direct(al, {q: runtime.direct_placement(ir, q) for q in range(R)}) == []
        n = 97 * R + 3
        xs = synth.inputs(R, n, "bfloat16", "intval")
        got = sim.simulate(al, xs, n, "bfloat16", "sum")
        ref = mpi_ref.allreduce(xs, "sum", "bfloat16")[0]
        for g in got:
            assert np.array_equal(nm.to_f64(g, "bfloat16"), ref)
