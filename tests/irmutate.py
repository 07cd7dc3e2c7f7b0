"""IR fault injection shared by the Python- and C++-validator tests."""
import copy

from paper_conf_asplos_cowanmmsx23_b200 import ir
from paper_conf_asplos_cowanmmsx23_b200 import programs as P


def _first_dep_step(a):
    for g in a.gpus:
        for tb in g.tbs:
            for st in tb.steps:
                if st.deps:
                    return g, tb, st
    raise AssertionError("program has no dependencies")


def mutations():
    """(name, expected rule, IR text) triples; every mutant must be rejected."""
    out = []
    ring = P.ring_allreduce(4)
    ap = P.allpairs_allreduce(4)

    a = copy.deepcopy(ring)
    del a.gpus[1].tbs[0].steps[2]
    for i, st in enumerate(a.gpus[1].tbs[0].steps):
        pass
    out.append(("drop_instruction", "V7", a))

    a = copy.deepcopy(ring)
    a.gpus[2].tbs[0].steps[0].cnt = 2
    out.append(("cnt_mismatch", "V7", a))

    a = copy.deepcopy(ap)
    g, tb, st = _first_dep_step(a)
    b, s = st.deps[0]
    g.tbs[b].steps[s].hasdep = False
    out.append(("cleared_hasdep", "V8", a))

    a = copy.deepcopy(ap)
    g, tb, st = _first_dep_step(a)
    st.deps = [(st.deps[0][0], 999)]
    out.append(("dep_missing_step", "V8", a))

    a = copy.deepcopy(ring)
    t = copy.deepcopy(a.gpus[0].tbs[0])
    t.id = 1
    t.recv = -1
    t.steps = [ir.Step("s", "i", 0, "-", -1, 1)]
    a.gpus[0].tbs.append(t)
    out.append(("duplicate_connection", "V5", a))

    a = copy.deepcopy(ring)
    a.gpus[0].tbs[0].send = 0
    out.append(("self_peer", "V4", a))

    a = copy.deepcopy(ring)
    for st in a.gpus[3].tbs[0].steps:
        if st.op == "rcs":
            st.dstbuf = "i"
            break
    out.append(("out_of_place_writes_input", "V3", a))

    a = copy.deepcopy(ring)
    a.gpus[0].tbs[0].steps[0].srcoff = 4
    out.append(("offset_out_of_range", "V6", a))

    a = copy.deepcopy(ring)
    a.gpus[2].i_chunks = 3
    a.gpus[2].o_chunks = 3
    out.append(("chunk_counts_differ", "V3", a))

    a = copy.deepcopy(ring)
    a.gpus[0].tbs[0].steps[0].op = "r"   # a recv where the send was: both sides wait
    a.gpus[0].tbs[0].steps[0].dstbuf, a.gpus[0].tbs[0].steps[0].dstoff = "o", 3
    out.append(("send_turned_recv", "V7", a))

    # cyclic dependency between two thread blocks of one rank
    a = copy.deepcopy(ap)
    g = a.gpus[0]
    t0, t1 = g.tbs[0], g.tbs[1]
    t0.steps[0].deps = [(t1.id, 0)]
    t1.steps[0].deps = [(t0.id, 0)]
    t0.steps[0].hasdep = t1.steps[0].hasdep = True
    out.append(("cyclic_dependency", "V9", a))

    a = copy.deepcopy(ring)
    a.ngpus = 5
    out.append(("ngpus_mismatch", "V2", a))

    return [(n, r, x.to_xml()) for n, r, x in out]


def too_many_tbs(limit):
    a = P.allpairs_allreduce(8, pair_tbs=False)
    return a.max_tbs() > limit, a.to_xml()


def outstanding_sends_ir():
    """Rank 0 posts 3 sends on channel 0 before (via a dependency) a send on channel 1
    that rank 1 waits for before it drains channel 0: needs >= 3 FIFO slots."""
    a = ir.Algo("outstanding3", "custom", 2, "Simple", False, 2, 1)
    g0 = ir.GpuProgram(0, 1, 1, 0)
    g0.tbs = [ir.ThreadBlock(0, 1, -1, 0, [ir.Step("s", "i", 0), ir.Step("s", "i", 0),
                                           ir.Step("s", "i", 0, hasdep=True)]),
              ir.ThreadBlock(1, 1, -1, 1, [ir.Step("s", "i", 0, deps=[(0, 2)])])]
    g1 = ir.GpuProgram(1, 1, 1, 0)
    g1.tbs = [ir.ThreadBlock(0, -1, 0, 0, [ir.Step("r", dstbuf="o", dstoff=0, deps=[(1, 0)]),
                                           ir.Step("r", dstbuf="o", dstoff=0), ir.Step("r", dstbuf="o", dstoff=0)]),
              ir.ThreadBlock(1, -1, 0, 1, [ir.Step("r", dstbuf="o", dstoff=0, hasdep=True)])]
    a.gpus = [g0, g1]
    return a.to_xml()


def recv_before_send_ir():
    a = ir.Algo("recvfirst", "custom", 2, "Simple", False, 1, 1)
    for q in range(2):
        g = ir.GpuProgram(q, 1, 1, 0)
        g.tbs = [ir.ThreadBlock(0, 1 - q, 1 - q, 0, [ir.Step("r", dstbuf="o", dstoff=0), ir.Step("s", "i", 0)])]
        a.gpus.append(g)
    return a.to_xml()


# ---------------------------------------------------------------- seeded random mutation
# (the C++ loader and the oracle's validator must return the same rule on
# random IR mutants, not only on hand-written ones.) One random edit per mutant: an attribute
# of a step / thread block / gpu / algo set to a value from a small adversarial domain, a
# step deleted / duplicated / swapped, a dependency redirected, or a thread block removed.
def random_bases():
    return [(P.ring_allreduce(4).to_xml(), 4), (P.allpairs_allreduce(4).to_xml(), 4),
            (P.ring_allgather(4, 1, 2).to_xml(), 4), (P.ring_reducescatter(4, 1, 1).to_xml(), 4),
            (P.alltoall_twostep(2, 2).to_xml(), 4), (P.hierarchical_allreduce(2, 2).to_xml(), 4),
            (P.ring_allreduce(4, inplace=True).to_xml(), 4), (P.oneshot_allreduce(4).to_xml(), 4),
            (P.nvls_allreduce(4, 2).to_xml(), 4), (P.nvls_allgather(4).to_xml(), 4),
            (P.ring_allreduce(4, channels=4, split_phases=True).to_xml(), 4),
            (P.ring_allreduce(4, rings=2).to_xml(), 4), (P.allpairs_allgather(4).to_xml(), 4)]


def mutate(text, rng):
    import xml.etree.ElementTree as ET
    root = ET.fromstring(text)
    gpus = list(root); g = rng.choice(gpus); tbs = list(g); tb = rng.choice(tbs); steps = list(tb)
    kind = rng.randrange(9)
    vals = ["-2", "-1", "0", "1", "2", "3", "4", "7", "65536", "x", "-"]
    if kind == 0 and steps:
        st = rng.choice(steps); a = rng.choice(["type","srcbuf","srcoff","dstbuf","dstoff","cnt","depid","deps","hasdep"])
        if a == "type": st.set(a, rng.choice(["s","r","cpy","re","rrc","rrs","rrcs","rcs","nop","zz","mrd","mst","mrs"]))
        elif a.endswith("buf"): st.set(a, rng.choice(["i","o","s","-","q"]))
        else: st.set(a, rng.choice(vals))
    elif kind == 1:
        tb.set(rng.choice(["send","recv","chan","id"]), rng.choice(vals[:8]))
    elif kind == 2:
        g.set(rng.choice(["i_chunks","o_chunks","s_chunks","id"]), rng.choice(vals[:9]))
    elif kind == 3 and steps:
        tb.remove(rng.choice(steps))
        for i, st in enumerate(list(tb)): st.set("s", str(i))
    elif kind == 4 and steps:
        st = rng.choice(steps); import copy; c = copy.deepcopy(st); tb.append(c)
        for i, st in enumerate(list(tb)): st.set("s", str(i))
    elif kind == 5 and len(steps) > 1:
        i, j = rng.sample(range(len(steps)), 2)
        for x in list(tb): tb.remove(x)
        steps[i], steps[j] = steps[j], steps[i]
        for k, st in enumerate(steps): st.set("s", str(k)); tb.append(st)
    elif kind == 6 and steps:
        st = rng.choice(steps); b = rng.randrange(len(tbs)); s = rng.randrange(4)
        st.set("depid", str(b)); st.set("deps", str(s))
    elif kind == 7:
        root.set(rng.choice(["ngpus","coll","proto","inplace"]), rng.choice(["1","2","4","5","allreduce","allgather","custom","LL","Simple","bogus"]))
    else:
        g.remove(tb)
    return ET.tostring(root, encoding="unicode")


def random_mutants(seed, n):
    """n (text, nranks) mutants from a seeded generator."""
    import random
    rng = random.Random(seed)
    bases = random_bases()
    out = []
    for _ in range(n):
        base, R = rng.choice(bases)
        out.append((mutate(base, rng), R))
    return out
