"""Seeded synthetic inputs shared by the tests, bench.py and the oracle legs.

Holds none of the method's arithmetic: it only draws per-rank buffers. Recipe (DESIGN.md
"Input recipe"): rank r draws from a generator seeded ``seed + r`` (default 20230325);

* ``uniform``  — uniform[-1, 1) drawn in fp64, cast (RNE) to the dtype — ML gradients,
                 the AllReduce workload;
* ``intval``   — integer-valued floats in [-8, 8]: every partial sum of <= 8 ranks is
                 exact in bf16/fp16/fp32, so any reduction order gives the same bits;
* ``int``      — integers uniform in [-2^20, 2^20) (no overflow at R = 8) for int dtypes;
* ``pattern``  — position code ``rank * 2^24 + (index mod 2^24)`` (int32) or random raw
                 bits (other dtypes) for the data-movement collectives, compared bitwise.

Arrays are numpy in the dtype's storage type (bf16 = uint16 bit patterns).
"""
import numpy as np

SEED = 20230325

_STORAGE = {"int8": np.int8, "uint8": np.uint8, "int32": np.int32, "uint32": np.uint32,
            "int64": np.int64, "uint64": np.uint64, "float16": np.float16, "float32": np.float32,
            "float64": np.float64, "bfloat16": np.uint16}


def _to_bf16_bits(x64):
    import torch
    return torch.from_numpy(np.ascontiguousarray(x64, dtype=np.float64)).to(torch.bfloat16).view(torch.int16) \
        .numpy().view(np.uint16)


def _cast(x64, dtype):
    if dtype == "bfloat16":
        return _to_bf16_bits(x64)
    return x64.astype(_STORAGE[dtype])


def rank_input(rank, n, dtype, dist="uniform", seed=SEED):
    g = np.random.default_rng(seed + rank)
    if dist == "uniform":
        return _cast(g.uniform(-1.0, 1.0, n), dtype)
    if dist == "intval":
        return _cast(g.integers(-8, 9, n).astype(np.float64), dtype)
    if dist == "int":
        st = _STORAGE[dtype]
        if st in (np.uint8, np.int8):
            return g.integers(np.iinfo(st).min, np.iinfo(st).max, n, endpoint=True).astype(st)
        lo = 0 if np.issubdtype(st, np.unsignedinteger) else -(1 << 20)
        return g.integers(lo, 1 << 20, n).astype(st)
    if dist == "pattern":
        if dtype in ("int32", "uint32"):
            return (rank * (1 << 24) + (np.arange(n) % (1 << 24))).astype(_STORAGE[dtype])
        w = np.dtype(_STORAGE[dtype]).itemsize
        return np.frombuffer(g.bytes(n * w), dtype=_STORAGE[dtype]).copy()
    raise ValueError(dist)


def inputs(R, n, dtype, dist="uniform", seed=SEED):
    """Per-rank input buffers (n elements each) for ranks 0..R-1."""
    return [rank_input(r, n, dtype, dist, seed) for r in range(R)]


# ---------------------------------------------------------------------------------------
# Counter-based generator: value(rank, i) is a pure function of (seed, rank, i), so the GPU
# can fill multi-GiB buffers directly while the oracle evaluates any sampled index on the
# host with the same integer arithmetic (torch int64 ops, identical on CPU and CUDA).
def _mix32(x):
    x = ((x ^ (x >> 16)) * 0x45D9F3B) & 0xFFFFFFFF
    x = ((x ^ (x >> 16)) * 0x45D9F3B) & 0xFFFFFFFF
    return x ^ (x >> 16)


def hashed(rank, idx, dtype, seed=SEED):
    """uniform[-1, 1) (24-bit grid, exact in fp32) cast RNE to `dtype`, for int64 index
    tensor `idx` (any device). Returns a torch tensor of `dtype` on idx's device."""
    import torch
    key = (idx + rank * 0x01000193 + seed) & 0xFFFFFFFF
    h = _mix32(_mix32(key) ^ 0x5BD1E995)
    u = (h >> 8).to(torch.float32) * (2.0 ** -23) - 1.0
    tdt = {"bfloat16": torch.bfloat16, "float16": torch.float16, "float32": torch.float32,
           "float64": torch.float64}[dtype]
    return u.to(tdt)


def hashed_numpy(rank, idx, dtype, seed=SEED):
    """Host copy of `hashed` at numpy indices, in the dtype's numpy storage type."""
    import torch
    t = hashed(rank, torch.from_numpy(np.asarray(idx, dtype=np.int64)), dtype, seed)
    if dtype == "bfloat16":
        return t.view(torch.int16).numpy().view(np.uint16)
    return t.numpy()
