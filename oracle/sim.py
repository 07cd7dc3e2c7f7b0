"""Plain CPU execution of an MSCCL-IR program (test infrastructure).

Follows the interpreter of §6.2 / Fig. 5 step by step, sequentially:

* every thread block runs its instruction list in order (instruction loop, Fig. 5
  line 12; "decodes instructions ... and executes them in-order" P:L1470-1473);
* the whole list is repeated once per tile (pipelining loop, Fig. 5 line 10, P:L1290;
  P:L1412-1432), tile t of every chunk before tile t+1 (reading R3);
* an instruction with dependencies waits until the named (thread block, step) has
  executed in the same tile iteration (Fig. 5 lines 14-16 and 24-27, P:L1294-1307;
  P:L1475-1485; monotone counter = reading R4);
* a connection (sender, receiver, channel) is a FIFO of `slots` messages: a send
  blocks while `slots` messages are outstanding, a receive blocks until a message is
  present (§6.1 "Remote Buffers"; communication edges P:L938-942);
  fused ops (rrs/rrcs/rcs) need both at once (they hold their incoming slot while
  pushing);
* op semantics are §4.2, see ``irparse.OPS``.

The abstract machine sweeps thread blocks round-robin; if a full sweep makes no
progress before every block finished, the program deadlocks (the system is monotone, so
the verdict does not depend on the sweep order). The per-element data work is done by
a *domain*: ``NumericDomain`` (real numpy buffers), ``symbolic.SymbolicDomain`` (chunk
labels) or ``NullDomain`` (no data; deadlock analysis only).
"""
from collections import deque

import numpy as np

from . import numerics as nm
from .geometry import Geometry, buffer_elems


class Deadlock(RuntimeError):
    pass


class NullDomain:
    def exec_piece(self, q, st, j, t, incoming):
        return None


class Machine:
    def __init__(self, algo, domain, slots=8, iters=1):
        self.algo = algo
        self.domain = domain
        self.slots = slots
        self.iters = iters
        self.tbs = []                 # (rank, TB)
        self.prog = {}                # (rank, tb id) -> completed steps (all tiles)
        self.nsteps = {}
        self.fifo = {}                # (src, dst, chan) -> deque of messages
        for g in algo.gpus:
            for tb in g.tbs:
                self.tbs.append((g.id, tb))
                self.prog[(g.id, tb.id)] = 0
                self.nsteps[(g.id, tb.id)] = len(tb.steps)
                if tb.send >= 0:
                    self.fifo.setdefault((g.id, tb.send, tb.chan), deque())
                if tb.recv >= 0:
                    self.fifo.setdefault((tb.recv, g.id, tb.chan), deque())
        self.executed = 0

    def _ready(self, q, tb, st, t):
        for (b, s) in st.deps:
            if self.prog[(q, b)] < t * self.nsteps[(q, b)] + s + 1:
                return False
        if st.recvs and not self.fifo[(tb.recv, q, tb.chan)]:
            return False
        if st.sends and len(self.fifo[(q, tb.send, tb.chan)]) >= self.slots:
            return False
        return True

    def _exec(self, q, tb, st, t):
        msg = self.fifo[(tb.recv, q, tb.chan)].popleft() if st.recvs else None
        out = []
        for j in range(st.cnt):
            inc = msg[j] if msg is not None else None
            out.append(self.domain.exec_piece(q, st, j, t, inc))
        if st.sends:
            self.fifo[(q, tb.send, tb.chan)].append(out)
        self.executed += 1

    def run(self):
        total = {k: n * self.iters for k, n in self.nsteps.items()}
        while True:
            progressed = False
            done = True
            for q, tb in self.tbs:
                key = (q, tb.id)
                n = self.nsteps[key]
                while self.prog[key] < total[key]:
                    t, s = divmod(self.prog[key], n)
                    st = tb.steps[s]
                    if not self._ready(q, tb, st, t):
                        break
                    self._exec(q, tb, st, t)
                    self.prog[key] += 1
                    progressed = True
                if self.prog[key] < total[key]:
                    done = False
            if done:
                return
            if not progressed:
                stuck = []
                for q, tb in self.tbs:
                    key = (q, tb.id)
                    if self.prog[key] < total[key]:
                        t, s = divmod(self.prog[key], self.nsteps[key])
                        stuck.append("rank %d tb %d step %d (tile %d, %s)"
                                     % (q, tb.id, s, t, tb.steps[s].op))
                raise Deadlock("no thread block can progress: " + "; ".join(stuck[:8]))


class NumericDomain:
    """Real per-rank buffers in/out/scratch; reading R1 decides element spans.

    Per piece, the element count processed is the smaller of the src and dst chunk
    lengths that the op touches locally (reading R2); incoming FIFO data shorter than
    that is "stale slot" garbage, modelled as poison.
    """

    def __init__(self, algo, inputs, count, dtype, op, tile_elems=None):
        self.algo = algo
        self.dtype = dtype
        self.op = op
        self.geo = Geometry(algo, count, nm.elem_bytes(dtype))
        R = algo.ngpus
        self.T = tile_elems if tile_elems else self.geo.E
        st = nm.storage(dtype)
        self.bufs = []
        for q in range(R):
            x = np.array(inputs[q], dtype=st, copy=True)
            assert x.size == buffer_elems(algo.coll, "i", R, count)
            if algo.inplace:
                o = x
            else:
                o = nm.poison(dtype, buffer_elems(algo.coll, "o", R, count))
            s = nm.poison(dtype, algo.gpus[q].s_chunks * self.geo.E)
            self.bufs.append({"i": x, "o": o, "s": s})

    def _len(self, buf, k):
        return self.geo.span(buf, k)[1]

    def _multimem(self, q, st, j, t):
        """mrd / mst / mrs (reading R23): the same chunk span on every rank's buffer."""
        L = min(self._len(st.srcbuf, st.srcoff + j), self._len(st.dstbuf, st.dstoff + j))
        a = t * self.T
        m = max(0, min(a + self.T, L) - a)
        s0 = self.geo.span(st.srcbuf, st.srcoff + j)[0] + a
        d0 = self.geo.span(st.dstbuf, st.dstoff + j)[0] + a
        if st.reads_all:
            v = nm.mreduce([b[st.srcbuf][s0:s0 + m].copy() for b in self.bufs], self.op, self.dtype)
        else:
            v = self.bufs[q][st.srcbuf][s0:s0 + m].copy()
        for p, b in enumerate(self.bufs):
            if st.writes_all or p == q:
                b[st.dstbuf][d0:d0 + m] = v
        return None

    def exec_piece(self, q, st, j, t, incoming):
        if st.multimem:
            return self._multimem(q, st, j, t)
        B = self.bufs[q]
        lens = []
        if st.reads_src:
            lens.append(self._len(st.srcbuf, st.srcoff + j))
        if st.writes_dst:
            lens.append(self._len(st.dstbuf, st.dstoff + j))
        L = min(lens)
        a = t * self.T
        m = max(0, min(a + self.T, L) - a)
        if st.recvs:
            x = incoming[:m]
            if x.size < m:
                x = np.concatenate([x, nm.poison(self.dtype, m - x.size)])
        if st.reads_src:
            s0 = self.geo.span(st.srcbuf, st.srcoff + j)[0] + a
            src = B[st.srcbuf][s0:s0 + m].copy()
        if st.writes_dst:
            d0 = self.geo.span(st.dstbuf, st.dstoff + j)[0] + a
        op = st.op
        if op == "s":
            v = src
        elif op == "r":
            v = x
        elif op == "cpy":
            v = src
        elif op == "re":
            v = nm.reduce(B[st.dstbuf][d0:d0 + m], src, self.op, self.dtype)
        elif op in ("rrc", "rrs", "rrcs"):
            v = nm.reduce(x, src, self.op, self.dtype)
        elif op == "rcs":
            v = x
        else:  # nop
            return None
        if st.writes_dst:
            B[st.dstbuf][d0:d0 + m] = v
        return v.copy() if st.sends else None

    def outputs(self):
        return [b["o"] for b in self.bufs]


def simulate(algo, inputs, count, dtype, op="sum", slots=8, slot_bytes=None, max_cnt=None):
    """Execute `algo` on per-rank host `inputs`; returns the per-rank output buffers.

    Whole-chunk mode (one pipeline iteration) unless `slot_bytes` is given, in which case
    the tile size and iteration count follow DESIGN.md reading R3.
    """
    if count == 0:
        return [np.array(x, copy=True) for x in inputs]
    tile = None
    iters = 1
    if slot_bytes is not None:
        if max_cnt is None:
            max_cnt = max([st.cnt for g in algo.gpus for tb in g.tbs for st in tb.steps] + [1])
        geo = Geometry(algo, count, nm.elem_bytes(dtype))
        tile, iters = geo.tile(slot_bytes, max_cnt)
    dom = NumericDomain(algo, inputs, count, dtype, op, tile_elems=tile)
    Machine(algo, dom, slots=slots, iters=iters).run()
    return dom.outputs()
