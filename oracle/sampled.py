"""Oracle values at sampled output positions (test / bench infrastructure).

For sizes the simulator cannot run in seconds, the AllReduce result at an element e is
still fixed by the program: the symbolic run (oracle/symbolic.py, §3.2) gives,
for every output chunk k, its reduction tree over input chunks; element e of chunk k is
that tree evaluated on element (e - k*E) of each leaf chunk, one rounding per (+)
(reading R6). The chunk size E follows reading R1 (oracle/geometry.py).
"""
import numpy as np

from . import numerics as nm
from .geometry import Geometry
from .symbolic import check


def _eval(tree, leafval, op, dtype):
    if tree[0] == "in":
        return leafval(tree[1], tree[2])
    if tree[0] == "m+":  # multimem fold over the ranks (reading R23): one rounding
        return nm.mreduce([_eval(x, leafval, op, dtype) for x in tree[1:]], op, dtype)
    _, a, b = tree
    return nm.reduce(_eval(a, leafval, op, dtype), _eval(b, leafval, op, dtype), op, dtype)


def reduction_at(algo, value_at, count, dtype, op, idx, rank=0):
    """Output of `rank` at output element indices `idx` (AllReduce / ReduceScatter programs).

    value_at(q, indices) -> numpy array (storage dtype) of rank q's input at `indices`.
    Output element e lies in output chunk k = e // E at position e - k*E (the output
    buffer is one block for both collectives, reading R1); a leaf (q, kk) of that chunk's
    tree is input chunk kk of rank q, whose span comes from the same geometry (for
    ReduceScatter the input holds R blocks, so kk = b*C_b + j starts at b*n + j*E).
    """
    assert algo.coll in ("allreduce", "reducescatter")
    trees = check(algo)
    geo = Geometry(algo, count, nm.elem_bytes(dtype))
    idx = np.asarray(idx, dtype=np.int64)
    out = np.empty(idx.size, dtype=nm.storage(dtype))
    k_of = idx // geo.E
    for k in np.unique(k_of):
        sel = np.nonzero(k_of == k)[0]
        pos = idx[sel] - k * geo.E

        def leaf(q, kk, pos=pos):
            return value_at(q, geo.span("i", kk)[0] + pos)
        out[sel] = _eval(trees[rank][int(k)], leaf, op, dtype)
    return out


def allreduce_at(algo, value_at, count, dtype, op, idx, rank=0):
    """Output of `rank` at element indices `idx` (AllReduce programs)."""
    assert algo.coll == "allreduce"
    return reduction_at(algo, value_at, count, dtype, op, idx, rank)
