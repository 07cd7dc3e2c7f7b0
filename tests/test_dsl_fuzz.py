"""Seeded random MSCCLang programs through the whole DSL lowering (tests/progfuzz.py).

For every program: it lowers (§4-§5: instruction generation, fusion, channels, instances,
thread blocks, dependencies), both validators accept the IR (V1-V9), the happens-before race
detector finds nothing (V10) -- also under the C++ loader's direct-placement marking -- and the oracle simulator computes exactly the program's
sequential meaning -- each written out chunk equals the int32 sum of the chunks the program's
copies and reduces combined into it, in program order (§3.1-3.3)."""
import numpy as np
import pytest

import progfuzz
import synth
from oracle import irparse, races, sim, validate
from paper_conf_asplos_cowanmmsx23_b200 import dsl
from paper_conf_asplos_cowanmmsx23_b200.dsl import Collective, Program, chunk


def _check(algo, R, C, meaning, seed, rt=None):
    text = algo.to_xml()
    al = irparse.parse(text)   # in-place programs: the simulator's out aliases in (reading R8)
    validate.validate(al, nranks=R, slots=8)
    if rt is not None:
        ok, msg = rt.validate(text, R, slots=8)
        assert ok, msg
        # the C++ loader's direct-placement marking (reading R15) is race free too (V10)
        marking = {q: rt.direct_placement(text, q) for q in range(R)}
        assert races.check_direct(al, marking, alias=algo.inplace) == [], seed
    assert races.find_races(al) == []
    n = 8 * C * 37
    xs = synth.inputs(R, n, "int32", "int", seed=seed)
    out = sim.simulate(al, xs, n, "int32", "sum")
    for (r, k), (lo, hi, v) in progfuzz.expected_out(meaning, xs, C, n).items():
        assert np.array_equal(out[r][lo:hi], v), (seed, r, k)


@pytest.fixture(scope="module")
def rt():
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    return runtime


@pytest.mark.parametrize("block", range(10))
def test_random_programs_lower_to_their_sequential_meaning(block, rt):
    for seed in range(block * 100, (block + 1) * 100):
        prog = progfuzz.random_program(seed)
        assert prog is not None, "seed %d: the DSL refused a sequential program" % seed
        _check(*prog, seed, rt)


def _lower(R, C, S, body, instances=1):
    with Program("pin", Collective(R, C, C), instances=instances) as p:
        body()
    return p.lower()


def test_reduce_into_its_second_operand():
    """c1.reduce(c2, buffer=c2's location): the result must be c1 (+) c2, not 2 c1 -- a copy
    of c1 into the destination before the reduce would overwrite c2 (found by the fuzzer)."""
    def body():
        chunk(0, "in", 1).copy(0, "sc", 0)
        chunk(0, "in", 0).reduce(chunk(0, "sc", 0), buffer="sc", index=0)
        chunk(0, "sc", 0).copy(0, "out", 0)
    algo = _lower(1, 2, 1, body)
    meaning = {(0, "o", 0): ((0, 0), (0, 1))}
    _check(algo, 1, 2, meaning, 5)
    steps = [st.op for tb in algo.gpus[0].tbs for st in tb.steps]
    assert "cpy" in steps and steps.count("re") == 1


def test_fifo_order_conflict_splits_the_connection():
    """Two messages on one connection whose receives depend on each other in the order
    opposite to the one the priority scheduler sends them (seed 3 of the fuzzer): lowering
    moves one message to another channel instead of failing."""
    prog = progfuzz.random_program(3, instances=1, inplace=False)
    assert prog is not None
    _check(*prog, 3)
    assert prog[0].nchannels >= 2


def test_shipped_programs_unchanged_by_conflict_handling():
    """The retry paths never trigger for the paper's programs: ring / all-pairs lower on the
    channels they ask for."""
    from paper_conf_asplos_cowanmmsx23_b200 import programs as P
    assert P.ring_allreduce(8).nchannels == 1
    assert P.ring_allreduce(8, channels=8).nchannels == 8
    assert P.allpairs_allreduce(8).nchannels == 1


def test_explicit_channels_against_the_receivers_order_lower_in_program_order():
    """Messages the program pinned to one channel (ch=) whose receives depend on each other
    against the scheduler's send order (fuzzer seeds 478 / 829): the connection keeps the
    program order instead of failing."""
    for seed in (478, 829, 1020, 1651):
        prog = progfuzz.random_program(seed, inplace=False)
        assert prog is not None, seed
        _check(*prog, seed)


def test_partly_overlapping_local_op_is_refused():
    """A count-2 copy on one rank from out[0:2] to out[1:3] reads a chunk the same op writes:
    the gather-then-scatter meaning of an op and the interpreter's chunk-by-chunk execution
    would differ, so the DSL refuses it."""
    with pytest.raises(dsl.DSLError, match="partly overlaps"):
        with Program("ovl", Collective(1, 3, 3)):
            chunk(0, "in", 0, 2).copy(0, "out", 0)
            chunk(0, "out", 0, 2).copy(0, "out", 1)


def test_validators_agree_on_deadlock_with_one_and_two_slots(rt):
    """V9 on random programs with 1 and 2 FIFO slots: the C++
    loader and the oracle's validator return the same verdict."""
    verdicts = set()
    for seed in range(400):
        algo, R, C, _ = progfuzz.random_program(seed)
        text = algo.to_xml()
        al = irparse.parse(text)
        for s in (1, 2):
            try:
                validate.validate(al, nranks=R, slots=s, iters=2)
                py = None
            except validate.ValidationError as e:
                py = str(e)[:2]
            ok, msg = rt.validate(text, R, slots=s)
            assert py == (None if ok else msg[:2]), (seed, s, py, msg)
            verdicts.add(py)
    assert None in verdicts and "V9" in verdicts   # both outcomes occur
