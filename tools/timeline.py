"""Per-CTA latency timeline of one small launch (needs a MSCCL_TIMELINE=1 build, chosen with
MSCCL_LIB): entry, prologue end and the end of every step of every thread block, in us from
the first CTA's entry. Usage: MSCCL_LIB=tools/variants/timeline.so python tools/timeline.py [program]"""
import ctypes, os, sys
os.environ["MSCCL_TRACE"] = "1"
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import synth
from paper_conf_asplos_cowanmmsx23_b200 import programs as P, runtime as rt

rt.lib.msccl_debug_trace.restype = ctypes.POINTER(ctypes.c_uint64)
R = 8
rt.set_param("MSCCL_THREADS", int(os.environ.get("THREADS", 256)))
n = int(os.environ.get("N", 512))
which = sys.argv[1] if len(sys.argv) > 1 else "oneshot"
proto = os.environ.get("PROTO", "LL")
algo = {"oneshot": lambda: P.oneshot_allreduce(R, protocol=proto),
        "allpairs": lambda: P.allpairs_allreduce(R, protocol=proto),
        "ring8": lambda: P.ring_allreduce(R, channels=8, protocol=proto),
        "ring": lambda: P.ring_allreduce(R, protocol=proto)}[which]()
ir = algo.to_xml()
comms = rt.Comm.virtual(R, 0)
dev = torch.device("cuda:0")
send = [synth.hashed(q, torch.arange(n, device=dev), "float16") for q in range(R)]
recv = [torch.empty_like(x) for x in send]
progs = [c.load(ir) for c in comms]
for it in range(20):
    with rt.group():
        for q in range(R):
            comms[q].run(progs[q], send[q], recv[q], n)
    torch.cuda.synchronize()
tr = np.ctypeslib.as_array(rt.lib.msccl_debug_trace(), shape=(4096, 32)).copy()
ntb = [p.info()["thread_blocks"] for p in progs]
if not tr[:sum(ntb), 0].all():
    sys.exit("no timeline recorded (not a MSCCL_TIMELINE build)")
t0 = min(tr[i, 0] for i in range(sum(ntb)))
cta = 0
ends = []
for q in range(R):
    for b in range(ntb[q]):
        row = tr[cta]
        steps = [(row[2 + s] - t0) / 1e3 for s in range(10) if row[2 + s]]
        if row[18]:
            steps += ["| t1"] + ["%6.2f" % ((row[18 + s] - t0) / 1e3) for s in range(10) if row[18 + s]]
        if row[13]:
            steps += ["waitret %.2f" % ((row[31] - t0) / 1e3), "firstload %.2f ok=%d v=%x tgt=%x" % ((row[27] - t0) / 1e3, row[28], row[29], row[30]),
                      "chain-start %.2f" % ((row[24] - t0) / 1e3), "depword %.2f" % ((row[25] - t0) / 1e3),
                      "own-dep %.2f" % ((row[16] - t0) / 1e3), "setup %.2f" % ((row[17] - t0) / 1e3),
                      "chain-deps %.2f" % ((row[13] - t0) / 1e3), "chain-data %.2f" % ((row[14] - t0) / 1e3)]
        ends.append((row[15] - t0) / 1e3)
        if q < 2 and (len(steps) > 1 or os.environ.get("ALL")):
            print("rank %d tb %2d  entry %6.2f  prologue %6.2f  steps %s  exit %6.2f" % (
                q, b, (row[0] - t0) / 1e3, (row[1] - t0) / 1e3, " ".join(x if isinstance(x, str) else "%6.2f" % x for x in steps),
                (row[15] - t0) / 1e3))
        cta += 1
for cta_i in (7, 14):
    w = tr[2048 + cta_i]
    print("cta %d per-thread wait returns:" % cta_i, " ".join("%d:%.2f" % (k, (w[k] - t0) / 1e3) for k in range(32) if w[k]))
slow = int(np.argmax(ends))
row = tr[slow]
print("slowest cta %d: prologue %.2f steps %s exit %.2f" % (slow, (row[1] - t0) / 1e3, " ".join(
    "%.2f" % ((row[2 + s] - t0) / 1e3) for s in range(10) if row[2 + s]), (row[15] - t0) / 1e3))
entries = [(tr[i, 0] - t0) / 1e3 for i in range(cta)]
print("ctas %d  entry spread %.2f us  last exit %.2f us  median exit %.2f us" % (
    cta, max(entries), max(ends), float(np.median(ends))))
