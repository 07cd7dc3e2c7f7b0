"""Structural validation of MSCCL-IR (test infrastructure; independent of the C++ loader).

Rules (the same spec the C++ loader implements separately):

V1 well-formed (known ops / buffers / protocol; steps numbered 0..n-1; unique tb ids)
V2 ngpus == number of <gpu> == communicator size, ids 0..R-1
V3 chunk counts fit the collective; an out-of-place program never writes 'i'
V4 peers in [0,R) minus self, or -1; channel >= 0; at most `max_tbs` thread blocks per GPU
   (all thread blocks are co-resident)
V5 a connection (src, dst, channel) has exactly one sending and one receiving thread block
   (§5)
V6 the op's role matches the thread block's peers; 1 <= cnt; off + cnt <= chunk count
V7 k-th send and k-th receive on a connection carry the same cnt; equal message counts
V8 deps name an existing (tb, step) of another thread block on the same GPU, and every
   referenced step sets hasdep (Fig. 5 lines 25-27)
V9 no deadlock in the abstract machine with the protocol's FIFO slot count, run for >= 2
   pipeline iterations (§5.2; §6.1)
V11 multimem ops (mrd/mst/mrs, reading R23) address only the i/o buffers, the program uses
   the Simple protocol, and the thread blocks that hold them have the same ids on every rank (their start/end group barrier
   pairs thread block b of every rank)
V10 (races=True) no happens-before race between instructions (oracle/races.py; §3.3
   P:L859-867, §5.2); with `marking` (the loader's direct placement) also none
   after the direct writes are moved to the sends
"""
from .irparse import BUFS
from .sim import Deadlock, Machine, NullDomain


class ValidationError(ValueError):
    pass


def _fail(rule, msg):
    raise ValidationError("%s: %s" % (rule, msg))


def validate(algo, nranks=None, slots=8, max_tbs=148, max_channels=64, iters=2, races=False, marking=None):
    R = algo.ngpus
    if nranks is not None and nranks != R:
        _fail("V2", "program is for %d ranks, communicator has %d" % (R, nranks))
    if len(algo.gpus) != R or sorted(g.id for g in algo.gpus) != list(range(R)):
        _fail("V2", "need exactly %d <gpu> elements with ids 0..%d" % (R, R - 1))
    algo.gpus.sort(key=lambda g: g.id)
    g0 = algo.gpus[0]
    for g in algo.gpus:
        if g.i_chunks != g0.i_chunks or g.o_chunks != g0.o_chunks:
            _fail("V3", "rank %d chunk counts differ from rank 0" % g.id)
    ci, co = g0.i_chunks, g0.o_chunks
    ok = {"allreduce": ci == co and ci >= 1,
          "allgather": co == R * ci and ci >= 1,
          "reducescatter": ci == R * co and co >= 1,
          "alltoall": ci == co and ci % R == 0 and ci >= R,
          "custom": ci == co and ci >= 1}[algo.coll]
    if not ok:
        _fail("V3", "chunk counts i=%d o=%d do not fit %s over %d ranks" % (ci, co, algo.coll, R))
    if algo.inplace and algo.coll not in ("allreduce", "custom"):
        _fail("V3", "in-place programs are only defined for allreduce/custom")

    sends, recvs = {}, {}
    for g in algo.gpus:
        if len(g.tbs) > max_tbs:
            _fail("V4", "rank %d has %d thread blocks > %d" % (g.id, len(g.tbs), max_tbs))
        ids = [tb.id for tb in g.tbs]
        if sorted(ids) != list(range(len(ids))):
            _fail("V1", "rank %d thread block ids must be 0..%d" % (g.id, len(ids) - 1))
        g.tbs.sort(key=lambda tb: tb.id)
        nchunks = {"i": g.i_chunks, "o": g.o_chunks, "s": g.s_chunks}
        for tb in g.tbs:
            where = "rank %d tb %d" % (g.id, tb.id)
            for p in (tb.send, tb.recv):
                if p != -1 and not (0 <= p < R and p != g.id):
                    _fail("V4", "%s: bad peer %d" % (where, p))
            if not (0 <= tb.chan < max_channels):
                _fail("V4", "%s: channel %d out of range" % (where, tb.chan))
            if tb.send >= 0:
                key = (g.id, tb.send, tb.chan)
                if key in sends:
                    _fail("V5", "connection %s has two sending thread blocks" % (key,))
                sends[key] = (g.id, tb)
            if tb.recv >= 0:
                key = (tb.recv, g.id, tb.chan)
                if key in recvs:
                    _fail("V5", "connection %s has two receiving thread blocks" % (key,))
                recvs[key] = (g.id, tb)
            for i, st in enumerate(tb.steps):
                w = "%s step %d" % (where, i)
                if st.s != i:
                    _fail("V1", "%s: steps must be numbered in order" % w)
                if st.sends and tb.send < 0:
                    _fail("V6", "%s: %s needs a send peer" % (w, st.op))
                if st.recvs and tb.recv < 0:
                    _fail("V6", "%s: %s needs a receive peer" % (w, st.op))
                if st.op != "nop" and st.cnt < 1:
                    _fail("V6", "%s: cnt must be >= 1" % w)
                for used, buf, off in ((st.reads_src, st.srcbuf, st.srcoff),
                                       (st.writes_dst, st.dstbuf, st.dstoff)):
                    if not used:
                        continue
                    if buf not in BUFS:
                        _fail("V6", "%s: bad buffer %r" % (w, buf))
                    lim = nchunks["i"] if (algo.inplace and buf == "o") else nchunks[buf]
                    if off < 0 or off + st.cnt > lim:
                        _fail("V6", "%s: chunks [%d,%d) exceed %s buffer of %d chunks"
                              % (w, off, off + st.cnt, buf, lim))
                if st.op == "re" and (st.dstbuf not in BUFS or st.srcbuf not in BUFS):
                    _fail("V6", "%s: reduce needs src and dst" % w)
                if st.writes_dst and st.dstbuf == "i" and not algo.inplace:
                    _fail("V3", "%s: out-of-place program writes the input buffer" % w)
                if st.multimem and ("s" in (st.srcbuf, st.dstbuf)):
                    _fail("V11", "%s: multimem op on the scratch buffer (per-rank sizes)" % w)
                for (b, s) in st.deps:
                    if b == tb.id:
                        _fail("V8", "%s: depends on its own thread block" % w)
                    if not (0 <= b < len(g.tbs)) or not (0 <= s < len(g.tbs[b].steps)):
                        _fail("V8", "%s: dependency (%d,%d) does not exist" % (w, b, s))
                    if not g.tbs[b].steps[s].hasdep:
                        _fail("V8", "%s: dependency (%d,%d) does not set hasdep" % (w, b, s))
    for key in set(sends) | set(recvs):
        if key not in sends or key not in recvs:
            _fail("V5", "connection %s has no %s" % (key, "receiver" if key in sends else "sender"))
        sc = [st.cnt for st in sends[key][1].steps if st.sends]
        rc = [st.cnt for st in recvs[key][1].steps if st.recvs]
        if len(sc) != len(rc):
            _fail("V7", "connection %s: %d sends vs %d receives" % (key, len(sc), len(rc)))
        for k, (a, b) in enumerate(zip(sc, rc)):
            if a != b:
                _fail("V7", "connection %s message %d: send cnt %d != recv cnt %d" % (key, k, a, b))
    mm = [sorted(tb.id for tb in g.tbs if any(st.multimem for st in tb.steps)) for g in algo.gpus]
    if any(mm) and algo.proto != "Simple":
        _fail("V11", "multimem programs use the Simple protocol")
    for g, ids in zip(algo.gpus, mm):
        if ids != mm[0]:
            _fail("V11", "rank %d holds multimem ops in thread blocks %s, rank 0 in %s" % (g.id, ids, mm[0]))
    try:
        Machine(algo, NullDomain(), slots=slots, iters=iters).run()
    except Deadlock as e:
        _fail("V9", "deadlock with %d FIFO slots: %s" % (slots, e))
    if races or marking is not None:
        from . import races as hb
        found = hb.find_races(algo, limit=1)
        if found:
            _fail("V10", "%r" % found[0])
        if marking is not None:
            try:
                found = hb.check_direct(algo, marking, limit=1)
            except hb.MarkingError as e:
                _fail("V10", "direct-placement marking: %s" % e)
            if found:
                _fail("V10", "with direct placement: %r" % found[0])
    return True
