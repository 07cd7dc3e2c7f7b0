"""Oracle-side MSCCL-IR reader (test infrastructure; see oracle/__init__.py).

MSCCL-IR is "a tree data structure that divides a collective into individual GPU
programs that are subdivided into thread blocks containing a list of instructions that
are sequentially executed" (§5; Fig. 4). A thread block has
at most one send peer and one receive peer plus a channel. An
instruction carries op, src/dst buffer and chunk offset, count and cross-thread-block
dependencies (Fig. 5 lines 1-5).

The concrete text syntax (attribute-only XML) is DESIGN.md reading R0; this parser is
written independently of the C++ loader in the product library.
"""
import xml.etree.ElementTree as ET
from dataclasses import dataclass, field

# op name -> (receives, sends, reads src, writes dst, reduces)
OPS = {
    "nop":  (False, False, False, False, False),
    "s":    (False, True,  True,  False, False),   # send(src)
    "r":    (True,  False, False, True,  False),   # recv(dst)
    "cpy":  (False, False, True,  True,  False),   # copy src -> dst
    "re":   (False, False, True,  True,  True),    # dst <- dst (+) src
    "rrc":  (True,  False, True,  True,  True),    # dst <- recv (+) src
    "rrs":  (True,  True,  True,  False, True),    # send(recv (+) src)
    "rrcs": (True,  True,  True,  True,  True),    # v = recv (+) src; dst <- v; send(v)
    "rcs":  (True,  True,  False, True,  False),   # v = recv; dst <- v; send(v)
    # multimem ops (reading R23): src/dst name the same chunk on
    # EVERY rank of the group (NVLS multicast address); no connection is used
    "mrd":  (False, False, True,  True,  True),    # dst_q <- (+)_p src_p            (ld_reduce)
    "mst":  (False, False, True,  True,  False),   # dst_p <- src_q for every p      (st)
    "mrs":  (False, False, True,  True,  True),    # v = (+)_p src_p; dst_p <- v     (ld_reduce + st)
}
MULTIMEM = ("mrd", "mst", "mrs")
BUFS = ("i", "o", "s")
COLLS = ("allreduce", "allgather", "reducescatter", "alltoall", "custom")
PROTOS = ("Simple", "LL", "LL128")


class IRError(ValueError):
    pass


@dataclass
class Step:
    s: int
    op: str
    srcbuf: str
    srcoff: int
    dstbuf: str
    dstoff: int
    cnt: int
    deps: list        # list of (tb, step)
    hasdep: bool

    @property
    def recvs(self):
        return OPS[self.op][0]

    @property
    def sends(self):
        return OPS[self.op][1]

    @property
    def reads_src(self):
        return OPS[self.op][2]

    @property
    def writes_dst(self):
        return OPS[self.op][3]

    @property
    def reduces(self):
        return OPS[self.op][4]

    @property
    def multimem(self):
        return self.op in MULTIMEM

    @property
    def reads_all(self):      # reads src on every rank
        return self.op in ("mrd", "mrs")

    @property
    def writes_all(self):     # writes dst on every rank
        return self.op in ("mst", "mrs")


@dataclass
class TB:
    id: int
    send: int
    recv: int
    chan: int
    steps: list = field(default_factory=list)


@dataclass
class GPU:
    id: int
    i_chunks: int
    o_chunks: int
    s_chunks: int
    tbs: list = field(default_factory=list)


@dataclass
class Algo:
    name: str
    coll: str
    ngpus: int
    proto: str
    inplace: bool
    nchannels: int
    gpus: list = field(default_factory=list)


def _int(el, key):
    v = el.get(key)
    if v is None:
        raise IRError("<%s> missing attribute %r" % (el.tag, key))
    try:
        return int(v)
    except ValueError:
        raise IRError("<%s> attribute %s=%r is not an integer" % (el.tag, key, v))


def _list(el, key):
    v = el.get(key, "-1")
    out = []
    for x in v.split(","):
        x = x.strip()
        if x == "":
            continue
        try:
            out.append(int(x))
        except ValueError:
            raise IRError("<%s> attribute %s=%r is not an integer list" % (el.tag, key, v))
    return out


def parse(text):
    """Parse IR text into an :class:`Algo`. Raises IRError on malformed input (rule V1)."""
    try:
        root = ET.fromstring(text)
    except ET.ParseError as e:
        raise IRError("not well-formed: %s" % e)
    if root.tag != "algo":
        raise IRError("root element must be <algo>")
    coll = root.get("coll")
    if coll not in COLLS:
        raise IRError("unknown collective %r" % coll)
    proto = root.get("proto", "Simple")
    if proto not in PROTOS:
        raise IRError("unknown protocol %r" % proto)
    algo = Algo(name=root.get("name", ""), coll=coll, ngpus=_int(root, "ngpus"), proto=proto,
                inplace=bool(_int(root, "inplace")), nchannels=int(root.get("nchannels", "1")))
    for g in root:
        if g.tag != "gpu":
            raise IRError("unexpected <%s> under <algo>" % g.tag)
        gpu = GPU(id=_int(g, "id"), i_chunks=_int(g, "i_chunks"), o_chunks=_int(g, "o_chunks"),
                  s_chunks=_int(g, "s_chunks"))
        for t in g:
            if t.tag != "tb":
                raise IRError("unexpected <%s> under <gpu>" % t.tag)
            tb = TB(id=_int(t, "id"), send=_int(t, "send"), recv=_int(t, "recv"), chan=_int(t, "chan"))
            for st in t:
                if st.tag != "step":
                    raise IRError("unexpected <%s> under <tb>" % st.tag)
                op = st.get("type")
                if op not in OPS:
                    raise IRError("unknown instruction type %r" % op)
                depid = _list(st, "depid")
                deps = _list(st, "deps")
                if len(depid) != len(deps):
                    raise IRError("depid/deps length mismatch")
                pairs = [(b, s) for b, s in zip(depid, deps) if b >= 0]
                for k in ("srcbuf", "dstbuf"):   # V1 "known enums" (DESIGN.md validator rules)
                    if st.get(k, "-") not in BUFS + ("-",):
                        raise IRError("unknown buffer %r" % st.get(k))
                tb.steps.append(Step(s=_int(st, "s"), op=op, srcbuf=st.get("srcbuf", "-"),
                                     srcoff=_int(st, "srcoff"), dstbuf=st.get("dstbuf", "-"),
                                     dstoff=_int(st, "dstoff"), cnt=_int(st, "cnt"), deps=pairs,
                                     hasdep=bool(_int(st, "hasdep"))))
            gpu.tbs.append(tb)
        algo.gpus.append(gpu)
    return algo
