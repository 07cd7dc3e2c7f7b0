"""MSCCL-IR in-memory model and text form (product side).

MSCCL-IR is a tree: program -> per-GPU program -> thread blocks (send peer, receive
peer, channel) -> ordered instructions (§5; Fig. 4). The
instruction fields follow Fig. 5 lines 1-5 and P:L1396-1410: op, src
buffer/offset, dst buffer/offset, count, dependencies (tb, step) and ``hasDep``.

Text syntax (reading R0)::

    <algo name coll ngpus proto inplace nchannels ninstances>
      <gpu id i_chunks o_chunks s_chunks>
        <tb id send recv chan>
          <step s type srcbuf srcoff dstbuf dstoff cnt depid deps hasdep/>

``type`` is one of nop s r cpy re rrc rrs rrcs rcs, or a multimem op mrd mst mrs (reading
R23); buffers are i/o/s ('-' = unused);
``depid``/``deps`` are equal-length comma lists ('-1' = none).
"""
from dataclasses import dataclass, field
import xml.etree.ElementTree as ET

OPCODES = {"nop": 0, "s": 1, "r": 2, "cpy": 3, "re": 4, "rrc": 5, "rrs": 6, "rrcs": 7, "rcs": 8,
           "mrd": 9, "mst": 10, "mrs": 11}
RECV_OPS = {"r", "rrc", "rrs", "rrcs", "rcs"}
SEND_OPS = {"s", "rrs", "rrcs", "rcs"}
SRC_OPS = {"s", "cpy", "re", "rrc", "rrs", "rrcs", "mrd", "mst", "mrs"}
DST_OPS = {"r", "cpy", "re", "rrc", "rrcs", "rcs", "mrd", "mst", "mrs"}
# multimem (NVLS) ops, reading R23: the same chunk on every rank of the group
MULTIMEM_OPS = {"mrd", "mst", "mrs"}


@dataclass
class Step:
    op: str
    srcbuf: str = "-"
    srcoff: int = -1
    dstbuf: str = "-"
    dstoff: int = -1
    cnt: int = 1
    deps: list = field(default_factory=list)
    hasdep: bool = False


@dataclass
class ThreadBlock:
    id: int
    send: int = -1
    recv: int = -1
    chan: int = 0
    steps: list = field(default_factory=list)


@dataclass
class GpuProgram:
    id: int
    i_chunks: int
    o_chunks: int
    s_chunks: int = 0
    tbs: list = field(default_factory=list)


@dataclass
class Algo:
    name: str
    coll: str
    ngpus: int
    proto: str = "Simple"
    inplace: bool = False
    nchannels: int = 1
    ninstances: int = 1
    gpus: list = field(default_factory=list)

    # ---- statistics used by docs / bench ----
    def max_tbs(self):
        return max(len(g.tbs) for g in self.gpus)

    def sends_per_rank(self):
        return [sum(1 for tb in g.tbs for st in tb.steps if st.op in SEND_OPS) for g in self.gpus]

    def to_xml(self):
        out = ['<algo name="%s" coll="%s" ngpus="%d" proto="%s" inplace="%d" nchannels="%d" ninstances="%d">'
               % (self.name, self.coll, self.ngpus, self.proto, int(self.inplace), self.nchannels,
                  self.ninstances)]
        for g in self.gpus:
            out.append('  <gpu id="%d" i_chunks="%d" o_chunks="%d" s_chunks="%d">'
                       % (g.id, g.i_chunks, g.o_chunks, g.s_chunks))
            for tb in g.tbs:
                out.append('    <tb id="%d" send="%d" recv="%d" chan="%d">' % (tb.id, tb.send, tb.recv, tb.chan))
                for s, st in enumerate(tb.steps):
                    depid = ",".join(str(b) for b, _ in st.deps) or "-1"
                    deps = ",".join(str(x) for _, x in st.deps) or "-1"
                    out.append('      <step s="%d" type="%s" srcbuf="%s" srcoff="%d" dstbuf="%s" dstoff="%d" '
                               'cnt="%d" depid="%s" deps="%s" hasdep="%d"/>'
                               % (s, st.op, st.srcbuf, st.srcoff, st.dstbuf, st.dstoff, st.cnt, depid, deps,
                                  int(st.hasdep)))
                out.append("    </tb>")
            out.append("  </gpu>")
        out.append("</algo>")
        return "\n".join(out) + "\n"


def from_xml(text):
    """Parse IR text back into :class:`Algo` (no validation; the C++ loader validates)."""
    root = ET.fromstring(text)
    a = Algo(name=root.get("name", ""), coll=root.get("coll"), ngpus=int(root.get("ngpus")),
             proto=root.get("proto", "Simple"), inplace=bool(int(root.get("inplace", "0"))),
             nchannels=int(root.get("nchannels", "1")), ninstances=int(root.get("ninstances", "1")))
    for g in root:
        gp = GpuProgram(int(g.get("id")), int(g.get("i_chunks")), int(g.get("o_chunks")),
                        int(g.get("s_chunks", "0")))
        for t in g:
            tb = ThreadBlock(int(t.get("id")), int(t.get("send")), int(t.get("recv")), int(t.get("chan")))
            for s in t:
                ids = [int(x) for x in s.get("depid", "-1").split(",") if x]
                sts = [int(x) for x in s.get("deps", "-1").split(",") if x]
                tb.steps.append(Step(s.get("type"), s.get("srcbuf", "-"), int(s.get("srcoff", "-1")),
                                     s.get("dstbuf", "-"), int(s.get("dstoff", "-1")), int(s.get("cnt", "1")),
                                     [(b, x) for b, x in zip(ids, sts) if b >= 0], bool(int(s.get("hasdep", "0")))))
            gp.tbs.append(tb)
        a.gpus.append(gp)
    return a
