"""Pins for oracle/races.py (happens-before race detection) and the
independent check of the loader's direct-placement marking (readings R15 / R15b).

What pins the detector to something other than itself:
* schedule independence: a program the detector calls race free gives bit-identical outputs
  under many random interleavings of the abstract machine (unbounded FIFOs); a program it
  flags (all-pairs with one dependency removed) gives different outputs under some
  interleaving -- the race is real;
* each dependency the lowering inserts into all-pairs is needed: removing
  any one of them is reported;
* hand-made racy programs: two thread blocks writing one output chunk; a direct receive
  whose destination an earlier instruction of its own thread block reads;
* the loader's marking (mscclDebugDirectPlacement, product code) is checked end to end:
  consistent on both ends of every connection, and race free with the writes moved to the
  sends, for every shipped program at R in {2,4,8} x instances in {1,2,4}.
"""
import random

import numpy as np
import pytest

import synth
from oracle import irparse, races, sim
from paper_conf_asplos_cowanmmsx23_b200 import programs as P


def _parse(a):
    return irparse.parse(a.to_xml() if hasattr(a, "to_xml") else a)


SHIPPED = {
    "ring": lambda R, r: P.ring_allreduce(R, instances=r),
    "ring_inplace": lambda R, r: P.ring_allreduce(R, instances=r, inplace=True),
    "ring_channels": lambda R, r: P.ring_allreduce(R, channels=R, instances=r),
    "ring_split": lambda R, r: P.ring_allreduce(R, channels=R, instances=r, split_phases=True),
    "ring_k2": lambda R, r: P.ring_allreduce(R, instances=r, rings=2),
    "ring_LL128": lambda R, r: P.ring_allreduce(R, instances=r, protocol="LL128"),
    "allpairs": lambda R, r: P.allpairs_allreduce(R, instances=r, protocol="Simple"),
    "oneshot": lambda R, r: P.oneshot_allreduce(R, instances=r, protocol="Simple"),
    "allgather": lambda R, r: P.ring_allgather(R, 1, r),
    "allgather_allpairs": lambda R, r: P.allpairs_allgather(R, r),
    "reducescatter": lambda R, r: P.ring_reducescatter(R, 1, r),
    "alltoall": lambda R, r: P.alltoall_twostep(1, R, r),
}


def _marking(ir, R):
    from paper_conf_asplos_cowanmmsx23_b200 import runtime  # the product library (no GPU needed)
    return {q: runtime.direct_placement(ir, q) for q in range(R)}


@pytest.mark.parametrize("R", [2, 4, 8])
@pytest.mark.parametrize("r", [1, 2, 4])
@pytest.mark.parametrize("name", sorted(SHIPPED))
def test_shipped_programs_race_free_with_loader_marking(name, R, r):
    algo = SHIPPED[name](R, r)
    ir = algo.to_xml()
    al = irparse.parse(ir)
    assert races.find_races(al) == []
    mk = _marking(ir, R)
    assert races.check_direct(al, mk) == [], "loader's direct placement races"


@pytest.mark.parametrize("prog", [P.hierarchical_allreduce(2, 2), P.hierarchical_allreduce(2, 4),
                                  P.hierarchical_allreduce(4, 2), P.alltoall_twostep(2, 4),
                                  P.alltoall_twostep(4, 2), P.alltonext(2, 4)],
                         ids=["hier2x2", "hier2x4", "hier4x2", "a2a2x4", "a2a4x2", "alltonext2x4"])
def test_hierarchical_programs_race_free(prog):
    ir = prog.to_xml()
    al = irparse.parse(ir)
    assert races.find_races(al) == []
    assert races.check_direct(al, _marking(ir, al.ngpus)) == []


def test_direct_placement_is_used():
    """The marking is not vacuous: the ring's allgather phase and the direct AllToAll place
    messages directly (counts of marked sends)."""
    for algo, R, want in ((P.ring_allreduce(8), 8, 8 * 7), (P.alltoall_twostep(1, 8), 8, 8 * 7)):
        mk = _marking(algo.to_xml(), R)
        assert sum(1 for q in mk for f, _, _ in mk[q] if f & 1) >= want


def test_every_loader_marked_receive_is_individually_safe():
    """Each receive the loader marks is safe on its own (marking only it and its sender)."""
    for algo, R in ((P.ring_allreduce(4, instances=2), 4), (P.allpairs_allreduce(4, protocol="Simple"), 4),
                    (P.alltonext(2, 2), 4)):
        ir = algo.to_xml()
        al = irparse.parse(ir)
        mk = _marking(ir, R)
        full = races.direct_map(al, mk)
        for e, v in full.items():
            if len(e) != 3:   # pulled-message entries (reading R30)
                continue
            kind, tgt = v
            if kind not in ("send", "both"):
                continue
            one = {e: ("send", tgt)}
            rq, rbuf, roff, _ = tgt
            for g in al.gpus:
                if g.id != rq:
                    continue
                for tb in g.tbs:
                    for s, st in enumerate(tb.steps):
                        if st.recvs and st.writes_dst and st.dstbuf == rbuf and st.dstoff == roff \
                                and full.get((rq, tb.id, s), ("",))[0] in ("recv", "both"):
                            one[(rq, tb.id, s)] = ("recv", None)
            assert races.find_races(al, direct=one) == [], e


def test_allpairs_every_dependency_is_needed():
    al = _parse(P.allpairs_allreduce(4))
    n = 0
    for g in al.gpus:
        for tb in g.tbs:
            for st in tb.steps:
                if not st.deps:
                    continue
                saved, st.deps = st.deps, []
                assert races.find_races(al, limit=1), "removing %s's deps must race" % (st,)
                st.deps = saved
                n += 1
    assert n >= 4 * 4


TWO_WRITERS = """<algo name="w2" coll="allgather" ngpus="2" proto="Simple" inplace="0" nchannels="1">
  <gpu id="0" i_chunks="1" o_chunks="2" s_chunks="0">
    <tb id="0" send="1" recv="-1" chan="0">
      <step s="0" type="s" srcbuf="i" srcoff="0" dstbuf="-" dstoff="-1" cnt="1" depid="-1" deps="-1" hasdep="0"/>
      <step s="1" type="cpy" srcbuf="i" srcoff="0" dstbuf="o" dstoff="1" cnt="1" depid="-1" deps="-1" hasdep="0"/>
    </tb>
    <tb id="1" send="-1" recv="1" chan="0">
      <step s="0" type="cpy" srcbuf="i" srcoff="0" dstbuf="o" dstoff="0" cnt="1" depid="-1" deps="-1" hasdep="0"/>
      <step s="1" type="r" srcbuf="-" srcoff="-1" dstbuf="o" dstoff="1" cnt="1" depid="-1" deps="-1" hasdep="0"/>
    </tb>
  </gpu>
  <gpu id="1" i_chunks="1" o_chunks="2" s_chunks="0">
    <tb id="0" send="-1" recv="0" chan="0">
      <step s="0" type="cpy" srcbuf="i" srcoff="0" dstbuf="o" dstoff="1" cnt="1" depid="-1" deps="-1" hasdep="0"/>
      <step s="1" type="r" srcbuf="-" srcoff="-1" dstbuf="o" dstoff="0" cnt="1" depid="-1" deps="-1" hasdep="0"/>
    </tb>
    <tb id="1" send="0" recv="-1" chan="0">
      <step s="0" type="s" srcbuf="i" srcoff="0" dstbuf="-" dstoff="-1" cnt="1" depid="-1" deps="-1" hasdep="0"/>
    </tb>
  </gpu>
</algo>"""


def test_two_thread_blocks_writing_one_chunk_race():
    rs = races.find_races(irparse.parse(TWO_WRITERS))
    assert rs and rs[0].loc == (0, "o", 1) and "w" in rs[0].kinds


def _direct_hazard_ir(dep):
    """Rank 1: thread block 0 copies o[0] -> s[0] and then receives into o[0] (program order
    makes that safe through the FIFO); thread block 1 copies o[0] -> o[1], ordered after the
    receive only when `dep`. Direct placement of the receive moves its write to rank 0's send,
    which nothing orders against thread block 0's earlier read."""
    d1 = 'depid="0" deps="1"' if dep else 'depid="-1" deps="-1"'
    return """<algo name="dh" coll="custom" ngpus="2" proto="Simple" inplace="0" nchannels="1">
  <gpu id="0" i_chunks="2" o_chunks="2" s_chunks="1">
    <tb id="0" send="1" recv="-1" chan="0">
      <step s="0" type="s" srcbuf="i" srcoff="0" dstbuf="-" dstoff="-1" cnt="1" depid="-1" deps="-1" hasdep="0"/>
    </tb>
  </gpu>
  <gpu id="1" i_chunks="2" o_chunks="2" s_chunks="1">
    <tb id="0" send="-1" recv="0" chan="0">
      <step s="0" type="cpy" srcbuf="o" srcoff="0" dstbuf="s" dstoff="0" cnt="1" depid="-1" deps="-1" hasdep="0"/>
      <step s="1" type="r" srcbuf="-" srcoff="-1" dstbuf="o" dstoff="0" cnt="1" depid="-1" deps="-1" hasdep="1"/>
    </tb>
    <tb id="1" send="-1" recv="-1" chan="0">
      <step s="0" type="cpy" srcbuf="o" srcoff="0" dstbuf="o" dstoff="1" cnt="1" %s hasdep="0"/>
    </tb>
  </gpu>
</algo>""" % d1


def test_hand_marked_direct_receive_with_earlier_reader_is_flagged():
    ir = _direct_hazard_ir(dep=True)
    al = irparse.parse(ir)
    assert races.find_races(al) == []        # FIFO semantics: ordered
    marking = {0: [(1, 1, 0)], 1: [(0, -1, -1), (2, -1, -1), (0, -1, -1)]}
    rs = races.check_direct(al, marking)
    assert rs and rs[0].loc == (1, "o", 0), rs
    # the loader does not mark it
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    assert all(f & 3 == 0 for f, _, _ in runtime.direct_placement(ir, 1))
    assert all(f & 3 == 0 for f, _, _ in runtime.direct_placement(ir, 0))


def test_unordered_reader_of_a_receive_destination_is_flagged():
    rs = races.find_races(irparse.parse(_direct_hazard_ir(dep=False)))
    assert rs and any(r.loc == (1, "o", 0) for r in rs)


def test_inconsistent_marking_rejected():
    ir = P.ring_allgather(2, 1, 1).to_xml()
    al = irparse.parse(ir)
    good = _marking(ir, 2)
    bad = {q: list(v) for q, v in good.items()}
    # clear the receive flag of rank 1's direct receive only
    k = next(i for i, (f, _, _) in enumerate(bad[1]) if f & 2)
    bad[1][k] = (bad[1][k][0] & ~2, -1, -1)
    with pytest.raises(races.MarkingError):
        races.direct_map(al, bad)


def test_aliasing_verdicts():
    """Out-of-place ring and all-pairs may be called in place (an 'aliassafe' IR attribute
    would be true); one-shot may not: its rank reads every peer's input chunk after a peer's
    broadcast may have overwritten it."""
    assert races.find_races(_parse(P.ring_allreduce(8, instances=2)), alias=True) == []
    assert races.find_races(_parse(P.allpairs_allreduce(8)), alias=True) == []
    assert races.find_races(_parse(P.oneshot_allreduce(8)), alias=True) != []


# ---------------------------------------------------------------- schedule independence
def _run_random_schedule(algo, xs, n, dtype, op, rng):
    """Execute with unbounded FIFOs, picking a random ready thread block at every step."""
    dom = sim.NumericDomain(algo, xs, n, dtype, op)
    m = sim.Machine(algo, dom, slots=1 << 30, iters=1)
    while True:
        ready = []
        for q, tb in m.tbs:
            key = (q, tb.id)
            if m.prog[key] < m.nsteps[key]:
                st = tb.steps[m.prog[key]]
                if m._ready(q, tb, st, 0):
                    ready.append((q, tb))
        if not ready:
            break
        q, tb = ready[rng.randrange(len(ready))]
        key = (q, tb.id)
        m._exec(q, tb, tb.steps[m.prog[key]], 0)
        m.prog[key] += 1
    assert all(m.prog[k] == m.nsteps[k] for k in m.prog), "stuck"
    return [o.copy() for o in dom.outputs()]


def test_race_free_means_schedule_independent():
    R, n = 4, 64
    xs = synth.inputs(R, n, "float32", "uniform")
    for algo in (P.allpairs_allreduce(R), P.ring_allreduce(R, instances=2), P.hierarchical_allreduce(2, 2)):
        al = _parse(algo)
        assert races.find_races(al) == []
        rng = random.Random(1)
        ref = _run_random_schedule(al, xs, n, "float32", "sum", rng)
        for _ in range(25):
            got = _run_random_schedule(al, xs, n, "float32", "sum", rng)
            assert all(np.array_equal(a.view(np.uint32), b.view(np.uint32)) for a, b in zip(ref, got))


def test_flagged_race_is_observable():
    """All-pairs with the dependency of its broadcast step removed: some interleaving sends
    the scratch chunk before the reduction finished, and the outputs differ."""
    R, n = 4, 64
    xs = synth.inputs(R, n, "float32", "uniform")
    al = _parse(P.allpairs_allreduce(R))
    victim = next(st for g in al.gpus for tb in g.tbs for st in tb.steps if st.deps and st.sends)
    victim.deps = []
    assert races.find_races(al, limit=1)
    rng = random.Random(2)
    outs = [_run_random_schedule(al, xs, n, "float32", "sum", rng) for _ in range(60)]
    distinct = {tuple(o.tobytes() for o in out) for out in outs}
    assert len(distinct) > 1


def test_validator_v10():
    from oracle import validate
    al = _parse(P.allpairs_allreduce(4))
    assert validate.validate(al, races=True)
    victim = next(st for g in al.gpus for tb in g.tbs for st in tb.steps if st.deps)
    victim.deps = []
    with pytest.raises(validate.ValidationError, match="^V10"):
        validate.validate(al, races=True)
    ir = _direct_hazard_ir(dep=True)
    with pytest.raises(validate.ValidationError, match="^V10"):
        validate.validate(irparse.parse(ir), marking={0: [(1, 1, 0)], 1: [(0, -1, -1), (2, -1, -1), (0, -1, -1)]})


def test_pulled_messages_marked_where_expected():
    """Reading R30: the loader pulls the first hop of every ReduceScatter chain (a plain send of
    an input chunk) in out-of-place Simple rings, on both ends of the connection, and nowhere
    in in-place or LL programs."""
    for algo, R, want in ((P.ring_allreduce(8), 8, 8), (P.ring_reducescatter(8, 1, 2), 8, 16),
                          (P.ring_allreduce(4, instances=2), 4, 8)):
        mk = _marking(algo.to_xml(), R)
        assert sum(1 for q in mk for f, _, _ in mk[q] if f & 8) == want
        assert sum(1 for q in mk for f, _, _ in mk[q] if f & 4) == want
    for algo, R in ((P.ring_allreduce(8, inplace=True), 8), (P.ring_allreduce(8, protocol="LL128"), 8),
                    (P.ring_allgather(8, 1, 1), 8)):
        mk = _marking(algo.to_xml(), R)
        assert not any(f & 12 for q in mk for f, _, _ in mk[q])


def test_a_pull_of_a_chunk_the_sender_rewrites_is_a_race():
    """The race checker models a pulled message as a read of the sender's input chunk at the
    receive: a hand-marked pull of a chunk the sender overwrites after its send (an in-place
    program, which the loader never pulls) is reported; the loader's own marking is race free."""
    from paper_conf_asplos_cowanmmsx23_b200.dsl import Collective, Program, chunk
    with Program("pull_war", Collective(2, 2, 2, inplace=True), protocol="Simple") as p:
        chunk(0, "in", 0).copy(1, "sc", 0)
        chunk(0, "in", 1).copy(0, "in", 0)
        chunk(1, "sc", 0).copy(1, "in", 1)
    ir = p.lower().to_xml()
    al = irparse.parse(ir)
    mk = _marking(ir, 2)
    assert not any(f & 12 for q in mk for f, _, _ in mk[q])
    assert races.check_direct(al, mk) == []
    forced = {q: list(v) for q, v in mk.items()}
    for q in (0, 1):
        for k, (f, b, o) in enumerate(forced[q]):
            st = [s for tb in al.gpus[q].tbs for s in tb.steps][k]
            if st.op == "s":
                forced[q][k] = (f | 8, b, o)
            elif st.op in ("r", "rcs", "rrc", "rrs", "rrcs"):
                forced[q][k] = (f | 4, b, o)
    assert races.check_direct(al, forced) != []
