"""MSCCLang DSL and its lowering to MSCCL-IR (product side).

The DSL is "embedded in Python as a traced DSL with a fluent API" (§3):
``chunk(rank, buffer, index, count)`` returns a reference; ``c.copy(rank, buffer,
index)`` and ``c1.reduce(c2)`` move chunks and return new references (Table 1,
P:L833-857). Only the latest reference to a location may be used and uninitialized
chunks may not be read.

Lowering follows §4-§5:

1. tracing records every copy/reduce in program order (Chunk DAG, §4.1);
2. each op expands into instructions — a remote copy into send + recv, a remote reduce
   into send + rrc, a local op into one instruction (§4.2); processing edges
   (true and false dependencies on buffer locations, per rank) and communication edges
   are recorded;
3. peephole fusion recv+send -> rcs (choosing the send on the longest path),
   rrc+send -> rrcs, rrcs whose local result is never used -> rrs (§4.3);
4. channel assignment: user ``ch=`` first, fused chains share one channel, everything
   else takes the lowest channel that keeps "at most one send and one receive
   connection per thread block" and "one sending and receiving thread block per
   connection" (§5; §5.2);
5. whole-program instances (the ``r`` of Fig. 8) replicate the program on
   interleaved sub-chunks with disjoint channels (reading R5);
6. thread-block assignment: priority (depth, reverse depth), one thread block per
   (send peer, receive peer, channel), heap-ordered global topological order, local ops
   to the thread block whose latest instruction is earliest (§5.2);
7. cross-thread-block processing edges become ``dep=(tb, step)`` + ``hasDep``
   (P:L1246-1260).

Extensions: ``c1.reduce(c2, buffer=, index=)`` names the destination of the
result (the rrc instruction already has separate src/dst), which lets
out-of-place programs keep the input buffer read-only; ``parallelize(k)`` splits each
op of a fragment into k ops of count/k on channels ch+i;
``c.multimem_reduce(...)`` / ``c.multimem_store(...)`` are the NVSwitch multicast ops of
reading R23 (not in the paper): one instruction on the issuing rank that
reads or writes the same chunks on EVERY rank.
"""
import heapq
from contextlib import contextmanager

from . import ir

BUFNAME = {"in": "i", "input": "i", "i": "i", "out": "o", "output": "o", "o": "o",
           "sc": "s", "scratch": "s", "s": "s"}


class DSLError(ValueError):
    pass


# ----------------------------------------------------------------------------- collectives
class Collective:
    coll = "custom"

    def __init__(self, num_ranks, i_chunks, o_chunks, inplace=False):
        self.num_ranks = num_ranks
        self.i_chunks = i_chunks
        self.o_chunks = o_chunks
        self.inplace = inplace


class AllReduce(Collective):
    """C chunks per rank; out_r[k] = sum_q in_q[k] (§3.2)."""
    coll = "allreduce"

    def __init__(self, num_ranks, chunks, inplace=False):
        super().__init__(num_ranks, chunks, chunks, inplace)


class AllGather(Collective):
    """`chunks` input chunks per rank; output block q holds rank q's input."""
    coll = "allgather"

    def __init__(self, num_ranks, chunks=1):
        super().__init__(num_ranks, chunks, num_ranks * chunks)


class ReduceScatter(Collective):
    """`chunks` output chunks per rank; input block r reduces into rank r's output."""
    coll = "reducescatter"

    def __init__(self, num_ranks, chunks=1):
        super().__init__(num_ranks, num_ranks * chunks, chunks)


class AllToAll(Collective):
    """chunk i on GPU j ends up on GPU i at index j (§7.3)."""
    coll = "alltoall"

    def __init__(self, num_ranks, chunks_per_peer=1):
        super().__init__(num_ranks, num_ranks * chunks_per_peer, num_ranks * chunks_per_peer)


class AllToNext(Collective):
    """GPU i sends its buffer to GPU i+1; the last sends nothing (§7.4)."""
    coll = "custom"

    def __init__(self, num_ranks, chunks=1):
        super().__init__(num_ranks, chunks, chunks)


# ----------------------------------------------------------------------------- tracing
_current = []


def _prog():
    if not _current:
        raise DSLError("no active Program (use `with Program(...):`)")
    return _current[-1]


class _TraceOp:
    __slots__ = ("kind", "src", "acc", "dst", "count", "ch")

    def __init__(self, kind, src, acc, dst, count, ch):
        self.kind, self.src, self.acc, self.dst, self.count, self.ch = kind, src, acc, dst, count, ch


class Ref:
    """Reference to `count` contiguous chunks of (rank, buffer, index) (Table 1)."""

    def __init__(self, prog, rank, buf, index, count, versions):
        self.prog, self.rank, self.buf, self.index, self.count = prog, rank, buf, index, count
        self.versions = versions

    def __repr__(self):
        return "Ref(rank=%d, %s[%d:%d])" % (self.rank, self.buf, self.index, self.index + self.count)

    def _check(self):
        cur = self.prog._versions(self.rank, self.buf, self.index, self.count)
        if cur != self.versions:
            raise DSLError("%r is not the latest reference to its chunks (P:L859-867)" % self)

    def copy(self, rank, buffer, index, ch=None):
        p = self.prog
        self._check()
        rank, index = p._rank(rank), p._index(index)
        b = BUFNAME[buffer]
        p._record("copy", (self.rank, self.buf, self.index), None, (rank, b, index), self.count, ch)
        return p._write(rank, b, index, self.count)

    def reduce(self, other, buffer=None, index=None, ch=None):
        """c1.reduce(c2): c1 <- c1 (+) c2 in place (Table 1); `buffer/index` extension
        names another destination on c1's rank."""
        p = self.prog
        self._check()
        other._check()
        if other.count != self.count:
            raise DSLError("reduce needs equal counts (%d vs %d)" % (self.count, other.count))
        b = self.buf if buffer is None else BUFNAME[buffer]
        idx = self.index if index is None else p._index(index)
        p._record("reduce", (other.rank, other.buf, other.index), (self.rank, self.buf, self.index),
                  (self.rank, b, idx), self.count, ch)
        return p._write(self.rank, b, idx, self.count)


    # ---- multimem (NVLS) ops, reading R23 ----
    def multimem_reduce(self, buffer, index=None, store_all=True, ch=None):
        """Reduce these chunks over every rank (the same buffer and index on each) and write
        the result to (buffer, index) on this rank (``mrd``) or on every rank (``mrs``).
        The sources must still hold the precondition's input on every rank, and results
        stored on other ranks are final (nothing may read them later): the group barrier of
        the multimem thread block orders only the multimem ops themselves."""
        p = self.prog
        p._mm_sources(self)
        b = BUFNAME[buffer]
        idx = self.index if index is None else p._index(index)
        p._record("mrs" if store_all else "mrd", (self.rank, self.buf, self.index), None, (self.rank, b, idx),
                  self.count, ch)
        if store_all:
            return p._mm_final(b, idx, self.count, self.rank)
        return p._write(self.rank, b, idx, self.count)

    def multimem_store(self, buffer, index, ch=None):
        """Store these chunks to (buffer, index) on every rank (``mst``); results are final."""
        p = self.prog
        self._check()
        b = BUFNAME[buffer]
        idx = p._index(index)
        p._record("mst", (self.rank, self.buf, self.index), None, (self.rank, b, idx), self.count, ch)
        return p._mm_final(b, idx, self.count, self.rank)


FINAL = -1  # version of a chunk written on a remote rank by a multimem op (reading R23)


def chunk(rank, buffer, index, count=1, sz=None):
    """Reference to the chunks currently at (rank, buffer, index) (Table 1)."""
    p = _prog()
    if sz is not None:
        count = sz
    rank, index = p._rank(rank), p._index(index)
    b = BUFNAME[buffer]
    vers = p._versions(rank, b, index, count)
    if any(v is None for v in vers):
        raise DSLError("chunk(%d, %s, %d, %d) accesses an uninitialized chunk (P:L847-848)"
                       % (rank, buffer, index, count))
    if any(v == FINAL for v in vers):
        raise DSLError("chunk(%d, %s, %d, %d) was written by a multimem op: multimem results are final "
                       "(reading R23)" % (rank, buffer, index, count))
    return Ref(p, rank, b, index, count, vers)


@contextmanager
def parallelize(k):
    """Split each op of the fragment into k ops on count/k chunks, channels ch+i."""
    p = _prog()
    p._par.append(k)
    try:
        yield
    finally:
        p._par.pop()


# ----------------------------------------------------------------------------- instructions
class _Ins:
    __slots__ = ("rank", "op", "src", "dst", "cnt", "sp", "rp", "ch", "seq", "deps", "raw", "succ",
                 "send_to", "recv_from", "dead", "tb", "step", "hasdep", "depth", "rdepth", "opi")

    def __init__(self, rank, op, src, dst, cnt, sp=-1, rp=-1, ch=None, seq=0):
        self.rank, self.op, self.src, self.dst, self.cnt = rank, op, src, dst, cnt
        self.sp, self.rp, self.ch, self.seq = sp, rp, ch, seq
        self.deps = set()      # processing edges (same rank): instructions this one waits for
        self.raw = set()       # subset of deps that are true (read-after-write) dependencies
        self.succ = set()      # reverse processing edges
        self.send_to = None    # communication edge: receiving instruction
        self.recv_from = None  # communication edge: sending instruction
        self.dead = False
        self.tb = None
        self.step = None
        self.hasdep = False
        self.opi = -1          # index of the traced op this instruction comes from


class _FifoConflict(Exception):
    """The scheduler cannot keep a connection FIFO-ordered: the receive at the head of the
    connection's queue waits (through processing edges) on a receive queued behind it."""

    def __init__(self, opis, conns):
        super().__init__(opis)
        self.opis = opis    # op indices of the messages involved, the queue head first
        self.conns = conns  # the connections whose queues are stuck


def _ch_ok(a, b):
    return a is None or b is None or a == b


class _ChainConflict(Exception):
    """A free fused chain fits no channel (it needs two connections on one thread block)."""


class Program:
    """Context in which a DSL program is traced and lowered (Fig. 2 architecture)."""

    def __init__(self, name, collective, protocol="Simple", instances=1, topology=None, pair_tbs=False):
        if protocol not in ("Simple", "LL", "LL128"):
            raise DSLError("unknown protocol %r" % protocol)
        self.pair_tbs = pair_tbs  # merge send-only (p,-1,ch) with recv-only (-1,p,ch) blocks (R17)
        self.name = name
        self.collective = collective
        self.protocol = protocol
        self.instances = instances
        self.topology = topology  # (N, G): rank/index tuples (n, g) -> n*G + g (§2)
        self.R = collective.num_ranks
        self._ver = {}
        for r in range(self.R):
            for k in range(collective.i_chunks):
                self._ver[(r, "i", k)] = 0
        self._ops = []
        self._par = []
        self._algo = None

    # --- context
    def __enter__(self):
        _current.append(self)
        return self

    def __exit__(self, *exc):
        _current.pop()
        return False

    # --- helpers
    def _rank(self, r):
        if isinstance(r, tuple):
            if not self.topology:
                raise DSLError("tuple ranks need Program(topology=(N, G))")
            n, g = r
            r = n * self.topology[1] + g
        if not 0 <= r < self.R:
            raise DSLError("rank %r out of range" % (r,))
        return r

    def _index(self, i):
        if isinstance(i, tuple):
            if not self.topology:
                raise DSLError("tuple indices need Program(topology=(N, G))")
            n, g = i
            return n * self.topology[1] + g
        return i

    def _key(self, rank, b, k):
        if b == "o" and self.collective.inplace:
            b = "i"
        return (rank, b, k)

    def _versions(self, rank, b, index, count):
        return tuple(self._ver.get(self._key(rank, b, k)) for k in range(index, index + count))

    def _write(self, rank, b, index, count):
        self._check_bounds(b, index, count)
        vers = []
        for k in range(index, index + count):
            key = self._key(rank, b, k)
            v = (self._ver.get(key) or 0) + 1
            self._ver[key] = v
            vers.append(v)
        return Ref(self, rank, b, index, count, tuple(vers))

    def _mm_sources(self, ref):
        """Multimem sources: the same chunks on every rank, still holding the input."""
        ref._check()
        for r in range(self.R):
            v = self._versions(r, ref.buf, ref.index, ref.count)
            if any(x != 0 for x in v):
                raise DSLError("multimem reduce of %s[%d:%d] needs the unmodified input on every rank "
                               "(rank %d's was written)" % (ref.buf, ref.index, ref.index + ref.count, r))

    def _mm_final(self, b, index, count, rank):
        self._check_bounds(b, index, count)
        # a store into another rank's chunk is ordered only against the other multimem ops (the
        # group barrier, reading R23): that chunk must not have been written there before
        for r in range(self.R):
            if r != rank and any(v is not None for v in self._versions(r, b, index, count)):
                raise DSLError("multimem store to %s[%d:%d] of rank %d, which the program already wrote "
                               "(reading R23: multimem stores go to chunks other ranks have not touched)"
                               % (b, index, index + count, r))
        for r in range(self.R):
            for k in range(index, index + count):
                self._ver[self._key(r, b, k)] = FINAL
        return None

    def _check_bounds(self, b, index, count):
        lim = {"i": self.collective.i_chunks, "o": self.collective.o_chunks}.get(b)
        if b == "o" and self.collective.inplace:
            lim = self.collective.i_chunks
        if index < 0 or (lim is not None and index + count > lim):
            raise DSLError("chunks [%d,%d) out of range for buffer %s" % (index, index + count, b))

    def _record(self, kind, src, acc, dst, count, ch):
        # an op reads its whole source before it writes (gather, then scatter: the oracle's and
        # the paper's chunk semantics) but the interpreter moves a count-c op chunk by chunk, so a
        # destination on the same rank and buffer that PARTLY overlaps an operand is ambiguous
        for opnd in (src, acc):
            if opnd is None or dst is None or opnd[0] != dst[0] or opnd[1] != dst[1]:
                continue
            lo = max(opnd[2], dst[2])
            hi = min(opnd[2], dst[2]) + count
            if lo < hi and opnd[2] != dst[2]:
                raise DSLError("%s: destination %s[%d:%d] partly overlaps an operand %s[%d:%d] on rank %d"
                               % (kind, dst[1], dst[2], dst[2] + count, opnd[1], opnd[2], opnd[2] + count,
                                  dst[0]))
        par = 1
        for k in self._par:
            par *= k
        if par == 1:
            self._ops.append(_TraceOp(kind, src, acc, dst, count, ch))
            return
        if count % par:
            raise DSLError("parallelize(%d) needs a count divisible by %d (got %d)" % (par, par, count))
        c = count // par
        for i in range(par):
            sh = lambda loc: None if loc is None else (loc[0], loc[1], loc[2] + i * c)
            self._ops.append(_TraceOp(kind, sh(src), sh(acc), sh(dst), c, (ch or 0) + i))

    # ------------------------------------------------------------------ lowering
    def lower(self, check_fusion=True):
        """Lower the traced program to an :class:`ir.Algo`.

        A connection is a FIFO (the k-th receive takes the k-th message), so the order in
        which the scheduler issues sends on a connection also orders their receives. When
        that order conflicts with the receiving rank's processing edges (the receive at the
        head of the queue waits on a receive behind it), the message at the head moves to a
        channel of its own and lowering restarts -- two connections, no FIFO relation
        (channels, §5.2). Shipped programs never need it."""
        forced = {}
        self._nch_seen = 1
        self._trace_conns = set()
        self._trace_all = False
        fuse = True
        for _ in range(4 * len(self._ops) + 8):
            try:
                ins = self._expand(forced)
                if fuse:
                    self._fuse(ins)
                ins = [x for x in ins if not x.dead]
                nch = self._assign_channels(ins)
                ins, nch = self._replicate(ins, nch)
                tbs = self._build_tbs(ins)
                self._schedule(ins, tbs)
                return self._emit(ins, tbs, nch)
            except _FifoConflict as e:
                # move a message the program left free (no explicit ch=) and not moved before
                movable = [i for i in e.opis if i >= 0 and self._ops[i].ch is None and i not in forced]
                if movable:
                    used = {op.ch for op in self._ops if op.ch is not None} | set(forced.values())
                    forced[movable[0]] = max(used | {self._nch_seen - 1}) + 1
                    continue
                # the program named these channels: keep its connections but send on them in
                # program (trace) order, which the sequential program itself proves schedulable
                new_conns = set(e.conns) - self._trace_conns
                if new_conns:
                    self._trace_conns |= new_conns
                elif not self._trace_all:
                    self._trace_all = True   # every connection in program order
                elif fuse:
                    fuse = False             # program order holds for the unfused instructions
                else:
                    raise DSLError("instruction DAG has a cycle")
            except _ChainConflict:
                # a fused chain (rcs / rrcs, §4.3) that passes one rank twice with different
                # peers needs two connections on its single channel: lower without fusion
                if not fuse:
                    raise DSLError("no channel satisfies the one-connection-per-thread-block rule")
                fuse = False
        raise DSLError("instruction DAG has a cycle")

    def ir(self):
        return self.lower().to_xml()

    # step 2: instruction generation (§4.2)
    def _expand(self, forced=None):
        ins = []
        seq = [0]
        cur = [0]

        def new(*a, **kw):
            if forced and cur[0] in forced and kw.get("ch") is None:
                kw["ch"] = forced[cur[0]]
            x = _Ins(*a, seq=seq[0], **kw)
            x.opi = cur[0]
            seq[0] += 1
            ins.append(x)
            return x

        for opi, op in enumerate(self._ops):
            cur[0] = opi
            s_r, s_b, s_i = op.src
            d_r, d_b, d_i = op.dst
            if op.kind in ir.MULTIMEM_OPS:  # one instruction on the issuing rank (reading R23)
                new(s_r, op.kind, (s_b, s_i), (d_b, d_i), op.count, ch=op.ch)
                continue
            if op.kind == "copy":
                if s_r == d_r:
                    new(s_r, "cpy", (s_b, s_i), (d_b, d_i), op.count, ch=op.ch)
                else:
                    a = new(s_r, "s", (s_b, s_i), None, op.count, sp=d_r, ch=op.ch)
                    b = new(d_r, "r", None, (d_b, d_i), op.count, rp=s_r, ch=op.ch)
                    a.send_to, b.recv_from = b, a
            else:
                a_r, a_b, a_i = op.acc
                if s_r == a_r:
                    if (s_b, s_i) == (d_b, d_i) and (a_b, a_i) != (d_b, d_i):
                        # the destination IS the second operand c2: dst <- dst (+) c1 (copying c1
                        # into dst first would overwrite c2 before it is read); (+) is
                        # commutative bit for bit (IEEE add / multiply, max / min up to NaN payloads)
                        new(a_r, "re", (a_b, a_i), (d_b, d_i), op.count, ch=op.ch)
                        continue
                    if (a_b, a_i) != (d_b, d_i):
                        new(a_r, "cpy", (a_b, a_i), (d_b, d_i), op.count, ch=op.ch)
                    new(a_r, "re", (s_b, s_i), (d_b, d_i), op.count, ch=op.ch)
                else:
                    a = new(s_r, "s", (s_b, s_i), None, op.count, sp=a_r, ch=op.ch)
                    b = new(a_r, "rrc", (a_b, a_i), (d_b, d_i), op.count, rp=s_r, ch=op.ch)
                    a.send_to, b.recv_from = b, a
        # processing edges: per rank, per chunk location, in trace order
        last_w, readers = {}, {}
        for x in ins:
            reads = []
            if x.src is not None:
                reads += [self._key(x.rank, x.src[0], x.src[1] + j) for j in range(x.cnt)]
            if x.op == "re":
                reads += [self._key(x.rank, x.dst[0], x.dst[1] + j) for j in range(x.cnt)]
            writes = [] if x.dst is None else [self._key(x.rank, x.dst[0], x.dst[1] + j) for j in range(x.cnt)]
            for loc in reads:
                w = last_w.get(loc)
                if w is not None:
                    x.deps.add(w)
                    x.raw.add(w)
            for loc in writes:
                w = last_w.get(loc)
                if w is not None:
                    x.deps.add(w)
                for rd in readers.get(loc, ()):
                    if rd is not x:
                        x.deps.add(rd)
            for loc in reads:
                readers.setdefault(loc, []).append(x)
            for loc in writes:
                last_w[loc] = x
                readers[loc] = []
            for d in x.deps:
                d.succ.add(x)
        self._final_writer = last_w
        return ins

    # step 3: fusion (§4.3)
    def _longest_from(self, ins):
        memo = {}
        order = sorted(ins, key=lambda x: -x.seq)
        for x in order:
            nxt = list(x.succ) + ([x.send_to] if x.send_to is not None else [])
            memo[x] = 1 + max([memo.get(y, 0) for y in nxt if not y.dead] + [0])
        return memo

    def _fuse(self, ins):
        longest = self._longest_from(ins)
        for x in ins:
            if x.dead or x.op not in ("r", "rrc"):
                continue
            # the fused instruction sits on one channel: the incoming connection's (x or its
            # sender named it) and the outgoing one's (s or its receiver) must not differ
            xch = x.ch if x.ch is not None else (x.recv_from.ch if x.recv_from is not None else None)
            cands = [s for s in x.succ if not s.dead and s.op == "s" and s.src == x.dst and s.cnt == x.cnt
                     and x in s.raw and s.deps == {x}
                     and _ch_ok(xch, s.ch if s.ch is not None else s.send_to.ch)]
            if not cands:
                continue
            s = max(cands, key=lambda c: (longest[c], -c.seq))
            x.op = "rcs" if x.op == "r" else "rrcs"
            x.sp = s.sp
            if x.ch is None:
                x.ch = s.ch
            x.send_to = s.send_to
            s.send_to.recv_from = x
            s.dead = True
            for y in s.succ:
                y.deps.discard(s)
                y.raw.discard(s)
                if y is not x:
                    y.deps.add(x)
                    x.succ.add(y)
            x.succ.discard(s)
        # rrcs whose local result is never used -> rrs
        outputs = {"o"} if not self.collective.inplace else {"i", "o"}
        for x in ins:
            if x.dead or x.op != "rrcs":
                continue
            used = any(x in y.raw for y in x.succ if not y.dead)
            if used:
                continue
            locs = [self._key(x.rank, x.dst[0], x.dst[1] + j) for j in range(x.cnt)]
            overwritten = all(self._final_writer.get(l) is not x for l in locs)
            if overwritten or locs[0][1] not in outputs:
                x.op = "rrs"
                x.dst = None

    # step 4: channels (§5.2)
    def _assign_channels(self, ins):
        parent = {}

        def find(a):
            while parent[a] is not a:
                parent[a] = parent[parent[a]]
                a = parent[a]
            return a

        edges = [x for x in ins if x.send_to is not None]
        for e in edges:
            parent[e] = e
        for x in ins:
            if x.recv_from is not None and x.send_to is not None:
                a, b = find(x.recv_from), find(x)
                if a is not b:
                    parent[b] = a
        groups = {}
        for e in edges:
            groups.setdefault(find(e), []).append(e)
        glist = sorted(groups.values(), key=lambda g: min(e.seq for e in g))
        fixed, free = [], []
        for g in glist:
            chs = {c for e in g for c in (e.ch, e.send_to.ch) if c is not None}
            if len(chs) > 1:
                if any(x.op in ("rcs", "rrcs", "rrs") for x in g):
                    raise _ChainConflict()   # fusion joined connections the program put on different channels
                raise DSLError("a fused chain mixes channels %s" % sorted(chs))
            (fixed if chs else free).append((g, chs.pop() if chs else None))
        self._tbstate = [_TBState() for _ in range(self.R)]
        for g, ch in fixed + free:
            members = set()
            for e in g:
                members.add(e)
                members.add(e.send_to)
            cands = [ch] if ch is not None else range(0, 4096)
            for c in cands:
                trial = [st.clone() for st in self._tbstate]
                if all(trial[m.rank].add(m.sp, m.rp, c) for m in members):
                    self._tbstate = trial
                    for m in members:
                        m.ch = c
                    break
            else:
                if ch is None or any(x.op in ("rcs", "rrcs", "rrs") for x in members):
                    raise _ChainConflict()   # retried without fusion (see lower)
                raise DSLError("no channel satisfies the one-connection-per-thread-block rule "
                               "(explicit ch=%s conflicts)" % ch)
        for x in ins:
            if x.ch is None:
                x.ch = 0
        nch = 1 + max([x.ch for x in ins if x.sp >= 0 or x.rp >= 0 or x.op in ir.MULTIMEM_OPS] + [0])
        self._nch_seen = max(getattr(self, "_nch_seen", 1), nch)
        return nch

    # step 5: whole-program instances (reading R5: interleaved sub-chunks)
    def _replicate(self, ins, nch):
        r = self.instances
        if r == 1:
            return ins, nch
        # chunk k of instance i becomes sub-chunk k*r + i; a count-c instruction therefore
        # becomes c count-1 instructions (its chunks are no longer contiguous).
        maxc = max([x.cnt for x in ins] + [1])
        out = []
        clones = {}
        for x in ins:
            for i in range(r):
                pieces = []
                for j in range(x.cnt):
                    m = lambda loc: None if loc is None else (loc[0], (loc[1] + j) * r + i)
                    y = _Ins(x.rank, x.op, m(x.src), m(x.dst), 1, x.sp, x.rp, x.ch + i * nch,
                             seq=(x.seq * r + i) * maxc + j)
                    y.opi = x.opi
                    pieces.append(y)
                    out.append(y)
                clones[(x, i)] = pieces
        for x in ins:
            for i in range(r):
                for j, y in enumerate(clones[(x, i)]):
                    y.deps = {p for d in x.deps for p in clones[(d, i)]}
                    y.raw = {p for d in x.raw for p in clones[(d, i)]}
                    y.succ = {p for d in x.succ for p in clones[(d, i)]}
                    if x.send_to is not None:
                        y.send_to = clones[(x.send_to, i)][j]
                    if x.recv_from is not None:
                        y.recv_from = clones[(x.recv_from, i)][j]
        return out, nch * r

    # step 6a: thread blocks = merged (send peer, recv peer, channel) tuples
    def _build_tbs(self, ins):
        states = [_TBState() for _ in range(self.R)]
        for x in sorted(ins, key=lambda x: x.seq):
            if x.sp >= 0 or x.rp >= 0:
                if not states[x.rank].add(x.sp, x.rp, x.ch):
                    raise DSLError("rank %d: (send %d, recv %d, ch %d) conflicts with an existing "
                                   "thread block" % (x.rank, x.sp, x.rp, x.ch))
        per_rank = [sorted({x.ch for x in ins if x.rank == r and x.op in ir.MULTIMEM_OPS}) for r in range(self.R)]
        mm_channels = per_rank[0] if per_rank else []
        if any(m != mm_channels for m in per_rank):
            raise DSLError("multimem ops must be issued on every rank on the same channels (their thread "
                           "blocks pair up across ranks, reading R23 / V11): %s" % per_rank)
        tbs = []
        for r in range(self.R):
            tuples = states[r].final()
            if self.pair_tbs:  # reading R17: one block per peer and channel for both directions
                recv_only = {(t[1], t[2]): t for t in tuples if t[0] < 0 <= t[1]}
                merged = []
                for t in tuples:
                    if t[0] >= 0 and t[1] < 0 and (t[0], t[2]) in recv_only:
                        merged.append((t[0], t[0], t[2]))
                        recv_only.pop((t[0], t[2]))
                    elif not (t[0] < 0 <= t[1]):
                        merged.append(t)
                tuples = merged + list(recv_only.values())
            lst = [_TB(t[0], t[1], t[2]) for t in tuples]
            # multimem ops run on their own thread block per channel, and that block must have
            # the same id on every rank (its group barrier pairs it with block b of every rank,
            # reading R23, rule V11): they come first, in channel order
            mm = [_TB(-1, -1, ch) for ch in mm_channels]
            lst = mm + lst
            if not lst and any(x.rank == r for x in ins):
                lst.append(_TB(-1, -1, 0))
            for i, tb in enumerate(lst):
                tb.id = i
            tbs.append(lst)
        return tbs

    # step 6b/7: priority, topological order, assignment, dependencies (§5.2)
    def _schedule(self, ins, tbs):
        preds = {x: set(x.deps) | ({x.recv_from} if x.recv_from is not None else set()) for x in ins}
        succs = {x: set() for x in ins}
        for x in ins:
            for p in preds[x]:
                succs[p].add(x)
        order = sorted(ins, key=lambda x: x.seq)
        for x in order:  # seq order is a topological order of the traced program
            x.depth = 1 + max([p.depth for p in preds[x]] + [-1])
        for x in reversed(order):
            x.rdepth = 1 + max([s.rdepth for s in succs[x]] + [-1])
        indeg = {x: len(preds[x]) for x in ins}
        heap = [(x.depth, -x.rdepth, x.seq, x) for x in ins if indeg[x] == 0]
        heapq.heapify(heap)
        pos = 0
        last = {}
        # a connection is a FIFO: its k-th receive must be the partner of its k-th send, so a
        # ready receive waits until every earlier-scheduled send's receive is scheduled.
        queue, deferred = {}, {}

        def conn(x):
            return (x.recv_from.rank, x.rank, x.ch)

        # connections that must carry their messages in program order (see lower)
        pend, held = {}, {}
        for x in sorted(ins, key=lambda x: x.seq):
            if x.send_to is not None and (getattr(self, "_trace_all", False)
                                          or conn(x.send_to) in getattr(self, "_trace_conns", ())):
                pend.setdefault(conn(x.send_to), []).append(x)

        while heap:
            _, _, _, x = heapq.heappop(heap)
            if x.send_to is not None and conn(x.send_to) in pend:
                if pend[conn(x.send_to)][0] is not x:
                    held.setdefault(conn(x.send_to), set()).add(x)
                    continue
            if x.recv_from is not None:
                q = queue[conn(x)]
                if q[0] is not x:
                    deferred.setdefault(conn(x), set()).add(x)
                    continue
                q.pop(0)
                if q and q[0] in deferred.get(conn(x), ()):
                    deferred[conn(x)].discard(q[0])
                    heapq.heappush(heap, (q[0].depth, -q[0].rdepth, q[0].seq, q[0]))
            if x.send_to is not None:
                queue.setdefault(conn(x.send_to), []).append(x.send_to)
                pq = pend.get(conn(x.send_to))
                if pq:
                    pq.pop(0)
                    if pq and pq[0] in held.get(conn(x.send_to), ()):
                        held[conn(x.send_to)].discard(pq[0])
                        heapq.heappush(heap, (pq[0].depth, -pq[0].rdepth, pq[0].seq, pq[0]))
            cands = [tb for tb in tbs[x.rank] if _fits(tb, x)]
            if not cands:
                raise DSLError("rank %d: no thread block for %s" % (x.rank, x.op))
            if x.sp >= 0 or x.rp >= 0:
                tb = cands[0]
            else:
                # a local op that depends on the last instruction of some thread block stays on
                # that block (program order replaces a cross-block dependency and keeps chains of
                # local reduces together, reading R16); otherwise the paper's rule: the block
                # whose latest instruction is earliest
                chained = [t for t in cands if t.ins and t.ins[-1] in x.deps]
                if chained:
                    tb = chained[0]
                else:
                    tb = min(cands, key=lambda t: (last.get(id(t), -1), t.id))
            x.tb, x.step = tb.id, len(tb.ins)
            tb.ins.append(x)
            last[id(tb)] = pos
            pos += 1
            for s in succs[x]:
                indeg[s] -= 1
                if indeg[s] == 0:
                    heapq.heappush(heap, (s.depth, -s.rdepth, s.seq, s))
        if pos != len(ins):
            stuck = [key for key, ds in deferred.items() if ds and queue.get(key)]
            stuck += [key for key, hs in held.items() if hs]
            if stuck:
                opis = []
                for key in stuck:
                    if queue.get(key):
                        opis.append(queue[key][0].opi)
                    opis += sorted(d.opi for d in deferred.get(key, ()))
                raise _FifoConflict(opis, stuck)
            raise DSLError("instruction DAG has a cycle")
        for x in ins:
            for d in x.deps:
                if d.tb != x.tb:
                    d.hasdep = True

    def _emit(self, ins, tbs, nch):
        c = self.collective
        r = self.instances
        scr = [0] * self.R
        for x in ins:
            for loc in (x.src, x.dst):
                if loc is not None and loc[0] == "s":
                    scr[x.rank] = max(scr[x.rank], loc[1] + x.cnt)
        algo = ir.Algo(self.name, c.coll, self.R, self.protocol, c.inplace, nch, r)
        for rank in range(self.R):
            g = ir.GpuProgram(rank, c.i_chunks * r, c.o_chunks * r, scr[rank])
            for tb in tbs[rank]:
                t = ir.ThreadBlock(tb.id, tb.send, tb.recv, tb.ch)
                for x in tb.ins:
                    dep = {}
                    for d in x.deps:
                        if d.tb != x.tb:
                            dep[d.tb] = max(dep.get(d.tb, -1), d.step)
                    sb, so = x.src if x.src is not None else ("-", -1)
                    db, do = x.dst if x.dst is not None else ("-", -1)
                    t.steps.append(ir.Step(x.op, sb, so, db, do, x.cnt, sorted(dep.items()), x.hasdep))
                g.tbs.append(t)
            algo.gpus.append(g)
        return algo


class _TB:
    def __init__(self, send, recv, ch):
        self.send, self.recv, self.ch = send, recv, ch
        self.ins = []
        self.id = -1


def _fits(tb, x):
    if x.op in ir.MULTIMEM_OPS:
        return tb.send == -1 and tb.recv == -1 and tb.ch == x.ch
    if x.sp >= 0 and (tb.send != x.sp or tb.ch != x.ch):
        return False
    if x.rp >= 0 and (tb.recv != x.rp or tb.ch != x.ch):
        return False
    return True


class _TBState:
    """Per-rank (send peer, recv peer, channel) tuples merged on shared connection ends."""

    def __init__(self):
        self.tbs = []    # [send, recv, ch] or None when merged away
        self.ends = {}   # ('s'|'r', peer, ch) -> tb index

    def clone(self):
        c = _TBState()
        c.tbs = [None if t is None else list(t) for t in self.tbs]
        c.ends = dict(self.ends)
        return c

    def add(self, sp, rp, ch):
        ts = self.ends.get(("s", sp, ch)) if sp >= 0 else None
        tr = self.ends.get(("r", rp, ch)) if rp >= 0 else None
        if sp >= 0 and rp >= 0:
            if ts is not None and tr is not None:
                if ts == tr:
                    return True
                a, b = self.tbs[ts], self.tbs[tr]
                if a[1] != -1 or b[0] != -1:
                    return False
                a[1] = rp
                self.ends[("r", rp, ch)] = ts
                self.tbs[tr] = None
                return True
            if ts is not None:
                if self.tbs[ts][1] != -1:
                    return False
                self.tbs[ts][1] = rp
                self.ends[("r", rp, ch)] = ts
                return True
            if tr is not None:
                if self.tbs[tr][0] != -1:
                    return False
                self.tbs[tr][0] = sp
                self.ends[("s", sp, ch)] = tr
                return True
            self.tbs.append([sp, rp, ch])
            self.ends[("s", sp, ch)] = self.ends[("r", rp, ch)] = len(self.tbs) - 1
            return True
        if sp >= 0:
            if ts is None:
                self.tbs.append([sp, -1, ch])
                self.ends[("s", sp, ch)] = len(self.tbs) - 1
            return True
        if rp >= 0:
            if tr is None:
                self.tbs.append([-1, rp, ch])
                self.ends[("r", rp, ch)] = len(self.tbs) - 1
            return True
        return True

    def final(self):
        return [tuple(t) for t in self.tbs if t is not None]
