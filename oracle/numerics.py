"""Element types and the per-instruction reduction (test infrastructure).

The paper only says reduce "applies a pre-defined reduction operation" (§4.2 P:L908-909,
"e.g., addition" P:L765-766). DESIGN.md reading R6: ops sum/prod/max/min; every
reduce / rrc / rrs / rrcs applies ONE binary op per element, rounded once (IEEE RNE) to
the buffer dtype; integers wrap modulo 2^bits. For bf16/fp16 this is computed as
round_RNE(fp32(a) op fp32(b)); for + and * that equals the correctly rounded narrow
result (fp32 has p' = 24 >= 2p+2 bits — pinned against exact rationals in
tests/test_oracle_numerics.py).

bf16 has no numpy type: it is stored as uint16 bit patterns and widened by a 16-bit
shift; narrowing is written out bit by bit below.
"""
import numpy as np

# NCCL numbering (nccl.h ncclDataType_t): name -> (id, storage dtype, bytes)
DTYPES = {
    "int8": (0, np.int8, 1), "uint8": (1, np.uint8, 1), "int32": (2, np.int32, 4),
    "uint32": (3, np.uint32, 4), "int64": (4, np.int64, 8), "uint64": (5, np.uint64, 8),
    "float16": (6, np.float16, 2), "float32": (7, np.float32, 4), "float64": (8, np.float64, 8),
    "bfloat16": (9, np.uint16, 2),
}
OPS = {"sum": 0, "prod": 1, "max": 2, "min": 3}
FLOATS = ("float16", "float32", "float64", "bfloat16")


def storage(dtype):
    return DTYPES[dtype][1]


def elem_bytes(dtype):
    return DTYPES[dtype][2]


def bf16_to_f32(u):
    """Exact widening: bf16 is the top half of an fp32 bit pattern."""
    return (np.asarray(u, dtype=np.uint16).astype(np.uint32) << 16).view(np.float32)


def f32_to_bf16(f):
    """Round-to-nearest-even narrowing of fp32 to bf16 (returns uint16 bit patterns)."""
    u = np.asarray(f, dtype=np.float32).view(np.uint32).astype(np.uint64)
    lsb = (u >> 16) & 1
    r = ((u + 0x7FFF + lsb) >> 16).astype(np.uint16)
    nan = np.isnan(np.asarray(f, dtype=np.float32))
    if nan.any():
        r = np.where(nan, np.uint16(0x7FC0), r)
    return r


def _apply(op, a, b):
    if op == "sum":
        return a + b
    if op == "prod":
        return a * b
    if op == "max":
        return np.maximum(a, b)
    if op == "min":
        return np.minimum(a, b)
    raise ValueError(op)


def reduce(a, b, op, dtype):
    """One element-wise binary reduction a (op) b in `dtype`, rounded once."""
    if dtype == "bfloat16":
        return f32_to_bf16(_apply(op, bf16_to_f32(a), bf16_to_f32(b)))
    if dtype == "float16":
        return _apply(op, a.astype(np.float32), b.astype(np.float32)).astype(np.float16)
    with np.errstate(over="ignore"):
        return _apply(op, a, b).astype(storage(dtype))  # ints wrap modulo 2^bits


def to_f64(x, dtype):
    if dtype == "bfloat16":
        return bf16_to_f32(x).astype(np.float64)
    return np.asarray(x).astype(np.float64)


def from_f64(x, dtype):
    """Cast an fp64 array to the dtype's storage (RNE) — used for input generation only."""
    if dtype == "bfloat16":
        return f32_to_bf16(np.asarray(x, dtype=np.float64).astype(np.float32))
    return np.asarray(x).astype(storage(dtype))


def poison(dtype, n):
    """Stand-in for stale FIFO / scratch contents (never a valid output)."""
    if dtype in ("float16", "float32", "float64"):
        return np.full(n, np.nan, dtype=storage(dtype))
    if dtype == "bfloat16":
        return np.full(n, 0x7FC1, dtype=np.uint16)
    return np.full(n, np.iinfo(storage(dtype)).max, dtype=storage(dtype))


# ---------------------------------------------------------------- multimem reduction (N2)
MULTIMEM_OPS = ("sum", "max", "min")


def mreduce(vals, op, dtype):
    """The value a multimem reduce returns for one element over the group's copies
    (reading R23): the ranks' values folded in ascending rank
    order; fp16/bf16 sums accumulate in fp32 and round ONCE to the dtype (the switch's
    .acc::f32 reduction), fp32/fp64 sums round per add in the dtype, integers wrap, max/min
    are exact. There is no multimem product (P:L908-909 names no operator; PTX multimem
    has add/min/max only), so prod is rejected."""
    if op not in MULTIMEM_OPS:
        raise ValueError("multimem reduction supports sum/max/min, not %r" % op)
    if dtype in ("bfloat16", "float16"):
        w = [bf16_to_f32(v) if dtype == "bfloat16" else np.asarray(v, dtype=np.float16).astype(np.float32)
             for v in vals]
        acc = w[0].copy()
        for x in w[1:]:
            acc = _apply(op, acc, x).astype(np.float32)
        return f32_to_bf16(acc) if dtype == "bfloat16" else acc.astype(np.float16)
    acc = np.asarray(vals[0], dtype=storage(dtype)).copy()
    for x in vals[1:]:
        with np.errstate(over="ignore"):
            acc = _apply(op, acc, np.asarray(x, dtype=storage(dtype))).astype(storage(dtype))
    return acc
