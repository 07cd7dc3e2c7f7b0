"""Seeded random MSCCLang programs (test infrastructure).

Each program is a random sequence of the DSL's chunk operations (Table 1) on a
custom collective: `copy` of a chunk to any rank's out / scratch chunk, and `reduce` of two
chunks into an out / scratch chunk on the first one's rank (c1.reduce(c2, buffer=, index=),
reading R11), always through the latest reference of each chunk (§3.3). Beside
the program the generator returns its sequential meaning: the value of every written chunk
as a set of (rank, input chunk) contributions, evaluated op by op in program order. The
tests lower the program (tracing, fusion, channels, thread blocks, dependencies: §4-§5) and
check that the IR computes exactly that meaning -- in the oracle simulator, and on the GPU.
int32 sums make the value of a chunk independent of the reduction order, so the check is
about the dataflow the lowering produces.
"""
import random

import contextlib

from paper_conf_asplos_cowanmmsx23_b200.dsl import Collective, DSLError, Program, chunk, parallelize


def random_program(seed, protocol="Simple", instances=None, inplace=None, max_ranks=4):
    """(algo, R, C, meaning) or None when the DSL refuses the random program. meaning maps
    (rank, 'o', index) -> sorted tuple of (rank, in index) contributions (with repeats).
    Ops move 1 or 2 consecutive chunks (count > 1: strided tiles, reading R3) and sometimes
    name a channel (ch=, §5.2); a destination that partly overlaps an operand on the same
    rank is avoided (the DSL refuses it)."""
    if inplace is None:   # a quarter of the programs are in place: 'out' is 'in' (reading R8)
        inplace = random.Random(seed ^ 0x5EED).random() < 0.25
    ib = "i" if inplace else "o"   # the buffer results land in
    rng = random.Random(seed)
    R = rng.choice([2, 3, 4]) if max_ranks == 4 else rng.randint(2, max_ranks)
    C = rng.choice([1, 2, 3, 4])
    S = rng.choice([0, 1, 2, 3])
    n_ops = rng.randint(3, 16)
    inst = instances if instances is not None else rng.choice([1, 1, 2])
    meaning = {}
    for r in range(R):
        for k in range(C):
            meaning[(r, "i", k)] = ((r, k),)

    def span(loc, cnt):
        return [(loc[0], loc[1], loc[2] + j) for j in range(cnt)]

    def overlaps(a, b, cnt):
        return a[0] == b[0] and a[1] == b[1] and a[2] != b[2] and abs(a[2] - b[2]) < cnt

    final = set()   # chunks a multimem store wrote on every rank: final (reading R23)
    try:
        with Program("fuzz_%d" % seed, Collective(R, C, C, inplace=inplace), protocol=protocol,
                     instances=inst) as p:
            for _ in range(n_ops):
                cnt = 2 if rng.random() < 0.3 else 1
                if protocol == "Simple" and not inplace and rng.random() < 0.12:   # multimem round (Simple)
                    # every rank issues one (their thread blocks pair up, reading R23 / V11):
                    # mrd on the same chunk everywhere, or mrs on a distinct chunk per rank
                    if C < cnt:
                        continue
                    if C >= R and rng.random() < 0.5:
                        base = rng.randrange(C)
                        ks = [(base + r) % C for r in range(R)]
                        # stores go to chunks no other rank wrote before (reading R23)
                        if cnt > 1 or any((q, "o", k) in meaning for r, k in enumerate(ks) for q in range(R)
                                          if q != r):
                            continue
                        for r, k in enumerate(ks):
                            chunk(r, "in", k).multimem_reduce("out", k, store_all=True)
                            v = tuple(sorted((q, k) for q in range(R)))
                            for q in range(R):
                                meaning[(q, "o", k)] = v
                                final.add((q, "o", k))
                    else:
                        k = rng.randrange(C - cnt + 1)
                        if any((q, "o", k + j) in final for q in range(R) for j in range(cnt)):
                            continue
                        for r in range(R):
                            chunk(r, "in", k, cnt).multimem_reduce("out", k, store_all=False)
                            for j in range(cnt):
                                meaning[(r, "o", k + j)] = tuple(sorted((q, k + j) for q in range(R)))
                    continue
                have = sorted(l for l in meaning if l not in final and
                              all(x in meaning and x not in final for x in span(l, cnt)))
                if not have:
                    continue
                b = rng.choice([ib] + (["s"] if S >= cnt else []))
                size = C if b in ("o", "i") else S
                if size < cnt:
                    continue
                ch = rng.choice([None, None, None, 0, 1, 2])
                # parallelize(2) splits a 2-chunk op into two 1-chunk ops on
                # channels ch, ch+1
                par = parallelize(2) if cnt == 2 and rng.random() < 0.4 else contextlib.nullcontext()
                if rng.random() < 0.5 or len(have) < 2:   # copy
                    src = rng.choice(have)
                    dst = (rng.randrange(R), b, rng.randrange(size - cnt + 1))
                    if dst == src or overlaps(src, dst, cnt) or any(x in final for x in span(dst, cnt)):
                        continue
                    with par:
                        chunk(src[0], _name(src[1]), src[2], cnt).copy(dst[0], _name(b), dst[2], ch=ch)
                    vals = [meaning[x] for x in span(src, cnt)]
                    for x, v in zip(span(dst, cnt), vals):
                        meaning[x] = v
                else:                                       # reduce c1 (+) c2 -> (c1.rank, b, di)
                    c1, c2 = rng.sample(have, 2)
                    dst = (c1[0], b, rng.randrange(size - cnt + 1))
                    if overlaps(c1, dst, cnt) or overlaps(c2, dst, cnt) or overlaps(c1, c2, cnt) or \
                            any(x in final for x in span(dst, cnt)):
                        continue
                    with par:
                        chunk(c1[0], _name(c1[1]), c1[2], cnt).reduce(chunk(c2[0], _name(c2[1]), c2[2], cnt),
                                                                        buffer=_name(b), index=dst[2], ch=ch)
                    vals = [tuple(sorted(meaning[x] + meaning[y])) for x, y in zip(span(c1, cnt), span(c2, cnt))]
                    for x, v in zip(span(dst, cnt), vals):
                        meaning[x] = v
        algo = p.lower()
    except DSLError:
        return None
    return algo, R, C, {(k[0], "o", k[2]): v for k, v in meaning.items() if k[1] == ib}


def _name(b):
    return {"i": "in", "o": "out", "s": "sc"}[b]


def expected_out(meaning, xs, C, n):
    """Per written out chunk (rank, index): (lo, hi, the int32 sum of its contributions).
    n must be a multiple of 4 C, so every chunk (reading R1) has the same E = n / C elements
    (a ragged chunk would only be partly overwritten by a copy from a longer one, reading R2)."""
    import numpy as np
    assert n % (4 * C) == 0
    E = n // C
    out = {}
    for (r, _, k), contrib in meaning.items():
        acc = np.zeros(E, dtype=np.int64)
        for (q, j) in contrib:
            acc += xs[q][j * E:(j + 1) * E].astype(np.int64)
        out[(r, k)] = (k * E, (k + 1) * E, (acc & 0xFFFFFFFF).astype(np.uint32).view(np.int32))
    return out
