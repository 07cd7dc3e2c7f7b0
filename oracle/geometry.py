"""Chunk geometry for the oracle (test infrastructure; see oracle/__init__.py).

The paper fixes only that "chunks ... represent contiguous spans of elements with a
uniform size" whose byte size "is abstract" until runtime (§2, §3.1
P:L246-250), that scratch is sized from the highest scratch index, and that
a chunk larger than a FIFO slot is split into tiles processed tile-by-tile across all
chunks (§6.2 "Pipelining"; Fig. 5 line 10).

Everything concrete below is DESIGN.md reading R1 (blocks / ragged chunks) and R3
(strided tiles). The CUDA path implements the same *rule* in its own code.
"""


def blocks(coll, buf, R):
    """Number of equal blocks a per-rank buffer divides into (reading R1)."""
    if buf == "i":
        return {"allreduce": 1, "allgather": 1, "reducescatter": R, "alltoall": R, "custom": 1}[coll]
    if buf == "o":
        return {"allreduce": 1, "allgather": R, "reducescatter": 1, "alltoall": R, "custom": 1}[coll]
    raise ValueError(buf)


def buffer_elems(coll, buf, R, n):
    return blocks(coll, buf, R) * n


def chunks_per_block(algo):
    g = algo.gpus[0]
    return g.i_chunks // blocks(algo.coll, "i", algo.ngpus)


def elems_per_chunk(n, cb, V):
    """E = ceil(n / C_b) rounded up to a multiple of V (16-byte vectors)."""
    if n == 0:
        return 0
    e = -(-n // cb)
    return -(-e // V) * V


class Geometry:
    """Element spans of (buffer, chunk index) for one call (reading R1)."""

    def __init__(self, algo, n, elem_bytes):
        self.R = algo.ngpus
        self.coll = algo.coll
        self.n = n
        self.V = max(1, 16 // elem_bytes)
        self.w = elem_bytes
        self.cb = chunks_per_block(algo)
        self.E = elems_per_chunk(n, self.cb, self.V)

    def span(self, buf, k):
        """(start element, length) of chunk k of buffer buf."""
        if buf == "s":
            return k * self.E, self.E
        b, j = divmod(k, self.cb)
        start = b * self.n + j * self.E
        length = max(0, min(self.E, self.n - j * self.E))
        return start, length

    def tile(self, slot_bytes, max_cnt):
        """(T, I): tile elements and pipeline iterations (reading R3)."""
        if self.E == 0:
            return 0, 0
        t = (slot_bytes // (max_cnt * self.w)) // self.V * self.V
        if t < self.V:
            raise ValueError("FIFO slot too small for count %d" % max_cnt)
        t = min(t, self.E)
        return t, -(-self.E // t)
