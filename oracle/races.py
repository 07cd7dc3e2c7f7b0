"""Happens-before race detection over MSCCL-IR (test infrastructure; see oracle/__init__.py).

SURVEY §8(c)(iii) / rule V10. The paper argues race freedom from two things: the DSL's
"latest reference" rule, which orders every use of a chunk after the instruction that
produced it (§3.3), and the lowering's dependency insertion, which turns each
such processing edge between thread blocks into a `dep` (§5.2). This module
checks the outcome on the IR itself, without trusting either step.

Events
------
One event per instruction (rank q, thread block b, step s) of one pipeline iteration. Its
accesses are whole chunks of rank q's buffers, following the op table of §4.2
(``irparse.OPS``): reads src, writes dst, and a local ``re`` also reads dst.
In an in-place program ``o`` is ``i``; ``alias=True`` does the same for an
out-of-place program called in place (reading R8).

Happens-before = transitive closure of
  * program order inside a thread block ("executes them in-order");
  * dependency edges dep=(b', s') -> (b, s) on one rank (Fig. 5 lines 14-16);
  * communication edges: the k-th send on a connection (src, dst, channel) happens before
    the k-th receive on it (one sending and one receiving thread block per
    connection).
FIFO-capacity edges (the (k-s)-th receive before the k-th send, §6.1) are
left out on purpose: the verdict then holds for every slot count s >= 1.

Multimem ops (mrd / mst / mrs, reading R23) read or write the same chunk on
EVERY rank. Their thread block b synchronises with thread block b of every other rank at
its start and its end (the group barrier of the runtime). So for every pair of ranks p, q,
the start of (p, b) happens before the first instruction of (q, b), and the last
instruction of (q, b) happens before the end of (p, b). Start and end are extra events
with no accesses.

One pipeline iteration is enough. Tiles of different iterations touch disjoint elements
(reading R3), and every edge goes forward in time: program order leads from tile t to
t+1, and dependency and message edges stay inside one tile (V7 makes the k-th message the
same instruction pair in every tile). So a path between two events of tile t never visits
another tile, and the tile-t happens-before relation is the one computed here.

Race: two events touch the same (rank, buffer, chunk), at least one writes, and neither
happens before the other.

Direct placement (readings R15 / R15b, the paper's future work P:L2615-2624)
moves a write. When a receive is direct, the matched send stores the message straight into
the receiver's destination chunk. The write therefore belongs to the SEND event, on the
receiver's memory, and the receive event no longer writes. A direct ``rcs`` still reads
its destination, because it forwards from there. ``check_direct`` takes the loader's
marking, exported by ``mscclDebugDirectPlacement`` and computed by product code in
validate.cpp. It checks that the marking is consistent on both ends of each connection,
then checks race freedom with the moved writes. That gives the optimisation a correctness
argument that does not live in the product.
"""
from collections import defaultdict, deque


class Race:
    def __init__(self, loc, a, b, kinds):
        self.loc = loc          # (rank, buffer, chunk)
        self.a, self.b = a, b   # events (rank, tb, step)
        self.kinds = kinds      # ("w", "r") etc.

    def __repr__(self):
        return "race on rank %d %s[%d]: %s %s vs %s %s" % (
            self.loc[0], self.loc[1], self.loc[2], self.kinds[0], self.a, self.kinds[1], self.b)


class HBCycle(RuntimeError):
    pass


def _canon(algo, buf, alias):
    if buf == "o" and (algo.inplace or alias):
        return "i"
    return buf


def _multimem_groups(algo):
    """thread block id -> [(rank, steps)] of the blocks that hold multimem ops."""
    out = defaultdict(list)
    for g in algo.gpus:
        for tb in g.tbs:
            if tb.steps and any(st.multimem for st in tb.steps):
                out[tb.id].append((g.id, len(tb.steps)))
    return out


def _events(algo):
    ev = []
    for g in algo.gpus:
        for tb in g.tbs:
            for s, st in enumerate(tb.steps):
                ev.append((g.id, tb.id, s))
    for b, members in _multimem_groups(algo).items():
        for (p, _) in members:
            ev += [("B", p, b), ("E", p, b)]
    return ev


def _connections(algo):
    """(src, dst, chan) -> (sending events, receiving events), each in program order."""
    conn = defaultdict(lambda: ([], []))
    for g in algo.gpus:
        for tb in g.tbs:
            for s, st in enumerate(tb.steps):
                if st.sends:
                    conn[(g.id, tb.send, tb.chan)][0].append((g.id, tb.id, s))
                if st.recvs:
                    conn[(tb.recv, g.id, tb.chan)][1].append((g.id, tb.id, s))
    return conn


def happens_before(algo):
    """Returns (events, index, anc) where anc[i] is a Python-int bitset of the events that
    happen before event i (strictly)."""
    ev = _events(algo)
    idx = {e: i for i, e in enumerate(ev)}
    succ = defaultdict(list)
    indeg = [0] * len(ev)

    def edge(a, b):
        succ[idx[a]].append(idx[b])
        indeg[idx[b]] += 1

    for g in algo.gpus:
        for tb in g.tbs:
            for s in range(1, len(tb.steps)):
                edge((g.id, tb.id, s - 1), (g.id, tb.id, s))               # program order
            for s, st in enumerate(tb.steps):
                for (b, s2) in st.deps:
                    edge((g.id, b, s2), (g.id, tb.id, s))                  # dependency
    for (sends, recvs) in _connections(algo).values():
        for a, b in zip(sends, recvs):
            edge(a, b)                                                     # k-th send -> k-th recv
    for b, members in _multimem_groups(algo).items():                     # group barriers (R23)
        for (p, n) in members:
            edge(("B", p, b), (p, b, 0))
            edge((p, b, n - 1), ("E", p, b))
            for (q, m) in members:
                if q != p:
                    edge(("B", p, b), (q, b, 0))
                    edge((q, b, m - 1), ("E", p, b))
    anc = [0] * len(ev)
    q = deque(i for i in range(len(ev)) if indeg[i] == 0)
    done = 0
    while q:
        i = q.popleft()
        done += 1
        for j in succ[i]:
            anc[j] |= anc[i] | (1 << i)
            indeg[j] -= 1
            if indeg[j] == 0:
                q.append(j)
    if done != len(ev):
        raise HBCycle("happens-before has a cycle (the program deadlocks even with unbounded FIFOs)")
    return ev, idx, anc


def accesses(algo, alias=False, direct=None):
    """Chunk accesses per event: {(q, tb, s): [(rank, buf, chunk, "r"|"w"), ...]}.

    direct: None, or {(q, tb, s): ("send", (rank, buf, off, cnt)) | ("recv", None)} -- the
    direct-placement transformation described in the module docstring -- plus, for pulled
    messages (reading R30), ((q, tb, s), "pulled"): True on the send (it reads nothing) and
    ((q, tb, s), "pull"): (sender, buf, off, cnt) on the receive (it reads the sender's chunk)."""
    acc = defaultdict(list)
    direct = direct or {}
    for g in algo.gpus:
        q = g.id
        for tb in g.tbs:
            for s, st in enumerate(tb.steps):
                e = (q, tb.id, s)
                if st.multimem:                        # the same chunk on every rank (R23)
                    for p in range(algo.ngpus):
                        for j in range(st.cnt):
                            if st.reads_all or p == q:
                                acc[e].append((p, _canon(algo, st.srcbuf, alias), st.srcoff + j, "r"))
                            if st.writes_all or p == q:
                                acc[e].append((p, _canon(algo, st.dstbuf, alias), st.dstoff + j, "w"))
                    continue
                if st.reads_src and (e, "pulled") not in direct:   # a pulled send reads nothing (R30)
                    for j in range(st.cnt):
                        acc[e].append((q, _canon(algo, st.srcbuf, alias), st.srcoff + j, "r"))
                pull = direct.get((e, "pull"))
                if pull is not None:                   # a pulled receive reads the sender's chunk
                    (pq, pbuf, poff, pcnt) = pull
                    for j in range(pcnt):
                        acc[e].append((pq, _canon(algo, pbuf, alias), poff + j, "r"))
                if st.op == "re":
                    for j in range(st.cnt):
                        acc[e].append((q, _canon(algo, st.dstbuf, alias), st.dstoff + j, "r"))
                if st.writes_dst:
                    d = direct.get(e)
                    recv_direct = d is not None and d[0] in ("recv", "both")
                    for j in range(st.cnt):
                        loc = (q, _canon(algo, st.dstbuf, alias), st.dstoff + j)
                        if recv_direct:
                            if st.op == "rcs":           # forwards from its destination
                                acc[e].append(loc + ("r",))
                        else:
                            acc[e].append(loc + ("w",))
                d = direct.get(e)
                if d is not None and d[0] in ("send", "both"):
                    (rq, rbuf, roff, rcnt) = d[1]
                    for j in range(rcnt):
                        acc[e].append((rq, _canon(algo, rbuf, alias), roff + j, "w"))
    return acc


def find_races(algo, alias=False, direct=None, limit=20):
    """All unordered conflicting access pairs (up to `limit`)."""
    ev, idx, anc = happens_before(algo)
    acc = accesses(algo, alias, direct)
    byloc = defaultdict(list)
    for e, lst in acc.items():
        for (rq, buf, ch, kind) in lst:
            byloc[(rq, buf, ch)].append((idx[e], kind))
    races = []
    for loc, lst in sorted(byloc.items()):
        for x in range(len(lst)):
            for y in range(x + 1, len(lst)):
                (i, ki), (j, kj) = lst[x], lst[y]
                if i == j or (ki == "r" and kj == "r"):
                    continue
                if (anc[j] >> i) & 1 or (anc[i] >> j) & 1:
                    continue
                races.append(Race(loc, ev[i], ev[j], (ki, kj)))
                if len(races) >= limit:
                    return races
    return races


class MarkingError(ValueError):
    pass


def direct_map(algo, marking):
    """Turn the loader's per-rank marking into the `direct` argument of accesses().

    marking: {rank: [(flags, rdst_buf, rdst_chunk), ...]} in (thread block, step) order;
    flags bit 0 = direct send, bit 1 = direct receive, bit 2 = pulled receive, bit 3 = pulled
    send (reading R30); rdst_buf 0/1/2 = i/o/s.
    Raises MarkingError when the two ends of a connection disagree."""
    bufs = ("i", "o", "s")
    flat = {}
    for g in algo.gpus:
        lst = marking[g.id]
        k = 0
        for tb in g.tbs:
            for s, st in enumerate(tb.steps):
                flat[(g.id, tb.id, s)] = lst[k]
                k += 1
        if k != len(lst):
            raise MarkingError("rank %d: marking has %d entries, program %d" % (g.id, len(lst), k))
    out = {}
    steps = {(g.id, tb.id, s): st for g in algo.gpus for tb in g.tbs for s, st in enumerate(tb.steps)}
    for (sends, recvs) in _connections(algo).values():
        for a, b in zip(sends, recvs):
            fa, rb_, ro = flat[a]
            fb = flat[b][0]
            sp, rp = bool(fa & 8), bool(fb & 4)
            if sp != rp:
                raise MarkingError("send %s pulled=%s but its receive %s pulled=%s" % (a, sp, b, rp))
            if sp:
                ss = steps[a]
                if ss.op != "s":
                    raise MarkingError("pulled send %s is a %s (only a plain send moves a chunk unchanged)"
                                       % (a, ss.op))
                out[(a, "pulled")] = True
                out[(b, "pull")] = (a[0], ss.srcbuf, ss.srcoff, ss.cnt)
            sd, rd = bool(fa & 1), bool(fb & 2)
            if sd != rd:
                raise MarkingError("send %s direct=%s but its receive %s direct=%s" % (a, sd, b, rd))
            if not sd:
                continue
            rs = steps[b]
            if rs.op not in ("r", "rcs"):
                raise MarkingError("direct receive %s is a %s (data must land unchanged)" % (b, rs.op))
            if (bufs[rb_], ro) != (rs.dstbuf, rs.dstoff):
                raise MarkingError("send %s targets %s[%d] but receive %s writes %s[%d]"
                                   % (a, bufs[rb_], ro, b, rs.dstbuf, rs.dstoff))
            prev = out.get(a)
            out[a] = ("both" if prev and prev[0] == "recv" else "send", (b[0], rs.dstbuf, rs.dstoff, rs.cnt))
            prevb = out.get(b)
            out[b] = ("both", prevb[1]) if prevb and prevb[0] == "send" else ("recv", None)
    for e, (f, _, _) in flat.items():
        if (f & 12) and (e, "pull") not in out and (e, "pulled") not in out:
            raise MarkingError("%s marked pulled but its connection partner is not" % (e,))
        if (f & 2) and e not in out:
            raise MarkingError("receive %s marked direct but no send on its connection is" % (e,))
    return out


def check_direct(algo, marking, alias=False, limit=20):
    """Races of the program under the given direct-placement marking ([] = race free)."""
    return find_races(algo, alias=alias, direct=direct_map(algo, marking), limit=limit)
