"""Symbolic execution of MSCCL-IR: collective postconditions (test infrastructure).

§3.1-3.2: chunks are *input* chunks identified by (rank, index),
*reduction* chunks "identified by the list of input chunks that combine to form" them,
or *uninitialized*; a collective's precondition gives each input index a unique input
chunk and its postcondition names, for each output index, the input or reduction chunk
it must hold. Accessing an uninitialized chunk is an error. Checking the
postcondition on a symbolic run is how MSCCLang "automatically validate[s] that a
prospective algorithm is correct".

Two labels are carried for every chunk:

* ``leaves`` — the sorted list (multiset) of input chunks folded into it; the
  postcondition compares these;
* ``tree`` — the reduction tree with the two children of every (+) put in a canonical
  order (IEEE + and * are commutative, so this is exactly what fixes the float bits);
  equal trees on all ranks prove the AllReduce / AllGather outputs are bitwise
  identical across ranks (reading R7).
"""
from .sim import Machine

UNINIT = None


class SymbolicError(RuntimeError):
    pass


def leaf(q, k):
    return ((("in", q, k),), ("in", q, k))


def combine(a, b):
    if a is UNINIT or b is UNINIT:
        raise SymbolicError("reduction reads an uninitialized chunk")
    leaves = tuple(sorted(a[0] + b[0]))
    x, y = sorted([a[1], b[1]], key=repr)
    return (leaves, ("+", x, y))


class SymbolicDomain:
    def __init__(self, algo):
        self.algo = algo
        self.bufs = []
        for g in algo.gpus:
            b = {}
            for k in range(g.i_chunks):
                b[("i", k)] = leaf(g.id, k)
            self.bufs.append(b)

    def _key(self, buf, k):
        if self.algo.inplace and buf == "o":
            buf = "i"
        return (buf, k)

    def get(self, q, buf, k):
        v = self.bufs[q].get(self._key(buf, k), UNINIT)
        if v is UNINIT:
            raise SymbolicError("rank %d reads uninitialized chunk %s[%d]" % (q, buf, k))
        return v

    def exec_piece(self, q, st, j, t, incoming):
        if st.op == "nop":
            return None
        if st.multimem:  # reading R23: the same chunk on every rank, folded in ascending rank order
            if st.reads_all:  # one multimem node: the fold is evaluated with one rounding
                vals = [self.get(p, st.srcbuf, st.srcoff + j) for p in range(len(self.bufs))]
                v = (tuple(sorted(sum((x[0] for x in vals), ()))), ("m+",) + tuple(x[1] for x in vals))
            else:
                v = self.get(q, st.srcbuf, st.srcoff + j)
            for p in range(len(self.bufs)):
                if st.writes_all or p == q:
                    self.bufs[p][self._key(st.dstbuf, st.dstoff + j)] = v
            return None
        if st.recvs and incoming is UNINIT:
            raise SymbolicError("rank %d receives an uninitialized chunk" % q)
        src = self.get(q, st.srcbuf, st.srcoff + j) if st.reads_src else None
        op = st.op
        if op in ("s", "cpy"):
            v = src
        elif op in ("r", "rcs"):
            v = incoming
        elif op == "re":
            v = combine(self.get(q, st.dstbuf, st.dstoff + j), src)
        else:  # rrc, rrs, rrcs
            v = combine(incoming, src)
        if st.writes_dst:
            self.bufs[q][self._key(st.dstbuf, st.dstoff + j)] = v
        return v if st.sends else None

    def out(self, q, k):
        return self.bufs[q].get(self._key("o", k), UNINIT)


def expected(algo, q, k):
    """Postcondition: the multiset of input chunks output chunk k of rank q must hold."""
    R = algo.ngpus
    g = algo.gpus[0]
    if algo.coll == "allreduce":
        return tuple(sorted(("in", p, k) for p in range(R)))
    if algo.coll == "allgather":
        cb = g.i_chunks
        p, j = divmod(k, cb)
        return (("in", p, j),)
    if algo.coll == "reducescatter":
        cb = g.o_chunks
        return tuple(sorted(("in", p, q * cb + k) for p in range(R)))
    if algo.coll == "alltoall":
        cb = g.i_chunks // R
        p, j = divmod(k, cb)
        return (("in", p, q * cb + j),)
    if algo.coll == "custom":  # AllToNext (§7.4)
        if q == 0:
            return None
        return (("in", q - 1, k),)
    raise ValueError(algo.coll)


def check(algo, slots=8, require_rank_identical=True):
    """Symbolically run `algo`; raise SymbolicError if the postcondition fails.

    Returns the per-rank list of output trees (useful for closed-form comparisons).
    """
    dom = SymbolicDomain(algo)
    Machine(algo, dom, slots=slots, iters=1).run()
    trees = []
    for g in algo.gpus:
        row = []
        for k in range(g.o_chunks):
            exp = expected(algo, g.id, k)
            got = dom.out(g.id, k)
            if exp is None:
                row.append(None)
                continue
            if got is UNINIT:
                raise SymbolicError("rank %d output chunk %d is uninitialized" % (g.id, k))
            if got[0] != exp:
                raise SymbolicError("rank %d output chunk %d holds %s, postcondition wants %s"
                                    % (g.id, k, got[0], exp))
            row.append(got[1])
        trees.append(row)
    if require_rank_identical and algo.coll in ("allreduce", "allgather"):
        for q in range(1, len(trees)):
            for k, t in enumerate(trees[q]):
                if t != trees[0][k]:
                    raise SymbolicError("output chunk %d differs in reduction order between rank 0 "
                                        "and rank %d (not bitwise rank-consistent)" % (k, q))
    return trees
