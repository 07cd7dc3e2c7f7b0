"""Brute-force collective definitions (test infrastructure).

These are the plain definitions the IR programs must implement:

* AllReduce — "all rank's output buffer are identical and contain the C reduction
  chunks (sum_r c^r_0, ..., sum_r c^r_C)" (§3.2): out_r[e] = (+)_q in_q[e].
* AllToAll — "chunk i on GPU j ends up on GPU i at index j" (§7.3):
  out_r[q*n + e] = in_q[r*n + e].
* AllGather / ReduceScatter — the postconditions of the two ring helpers of Fig. 3b
   generalised to one block per rank (reading R1, R8):
  out_r[q*n + e] = in_q[e];   out_r[e] = (+)_q in_q[r*n + e].
* AllToNext — "GPU i sends a buffer of data to GPU i + 1, with the last GPU sending
  nothing" (§7.4): out_{i+1} = in_i.

Floating-point reductions are computed in fp64 (no rounding until the caller compares);
integer reductions exactly in Python integers, then wrapped modulo 2^bits.
"""
import numpy as np

from . import numerics as nm


def _wrap(vals, dtype):
    bits = 8 * nm.elem_bytes(dtype)
    signed = dtype.startswith("int")
    out = []
    for v in vals:
        v %= (1 << bits)
        if signed and v >= (1 << (bits - 1)):
            v -= (1 << bits)
        out.append(v)
    return np.array(out, dtype=nm.storage(dtype))


def _fold(arrays, op, dtype):
    """(op) over a list of same-length arrays: fp64 for floats, exact ints otherwise."""
    if dtype in nm.FLOATS:
        xs = np.stack([nm.to_f64(a, dtype) for a in arrays])
        if op == "sum":
            return xs.sum(axis=0)
        if op == "prod":
            return xs.prod(axis=0)
        if op == "max":
            return xs.max(axis=0)
        if op == "min":
            return xs.min(axis=0)
        raise ValueError(op)
    cols = [[int(v) for v in a] for a in arrays]
    res = []
    for e in range(len(cols[0]) if cols else 0):
        acc = cols[0][e]
        for c in cols[1:]:
            x = c[e]
            if op == "sum":
                acc = acc + x
            elif op == "prod":
                acc = acc * x
            elif op == "max":
                acc = max(acc, x)
            elif op == "min":
                acc = min(acc, x)
        res.append(acc)
    return _wrap(res, dtype)


def allreduce(inputs, op, dtype):
    r = _fold(inputs, op, dtype)
    return [r.copy() for _ in inputs]


def allgather(inputs):
    cat = np.concatenate(inputs)
    return [cat.copy() for _ in inputs]


def reducescatter(inputs, n, op, dtype):
    R = len(inputs)
    return [_fold([x[r * n:(r + 1) * n] for x in inputs], op, dtype) for r in range(R)]


def alltoall(inputs, n):
    R = len(inputs)
    return [np.concatenate([inputs[q][r * n:(r + 1) * n] for q in range(R)]) for r in range(R)]


def alltonext(inputs):
    """out_{i+1} = in_i; rank 0's output is unspecified (returned as None)."""
    R = len(inputs)
    return [None] + [inputs[i].copy() for i in range(R - 1)]
