"""AllReduce / AllToAll size sweep on 8 virtual ranks (BASELINE config 2/3/4 shapes on one GPU).

For every size and candidate program: device time per call (CUDA-graph replay for small
sizes, events around back-to-back calls for large), busBW, and bit-exact sampled parity of
the last call. Prints JSON lines and writes a markdown table (argv[1])."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch
import bench, synth
from oracle import irparse, sampled
from paper_conf_asplos_cowanmmsx23_b200 import programs as P, runtime as rt

R = 8
rt.set_param("MSCCL_THREADS", 256)
rt.set_param("MSCCL_SLOT_BYTES", 262144)
rt.set_param("MSCCL_MAX_CHANNELS", 64)
comms = rt.Comm.virtual(R, 0)
dev = torch.device("cuda:0")
stream = torch.cuda.current_stream()
SET = os.environ.get("SWEEP_SET", "base")
cands = [
    ("oneshot_LL", P.oneshot_allreduce(R, protocol="LL"), 1 << 20),
    ("allpairs_LL", P.allpairs_allreduce(R, protocol="LL"), 8 << 20),
    ("ring_ch8_LL", P.ring_allreduce(R, channels=8, protocol="LL"), 8 << 20),
    ("ring_ch8_LL128", P.ring_allreduce(R, channels=8, protocol="LL128"), 64 << 20),
    ("ring_ch8_i2_Simple", P.ring_allreduce(R, channels=8, instances=2), 1 << 30),
    ("ring_ch1_i32_Simple", P.ring_allreduce(R, instances=32), 1 << 30),
]
if SET == "mid":
    cands = [
        ("allpairs_i1_Simple", P.allpairs_allreduce(R, protocol="Simple"), 64 << 20),
        ("allpairs_i2_Simple", P.allpairs_allreduce(R, instances=2, protocol="Simple"), 64 << 20),
        ("allpairs_i2_LL128", P.allpairs_allreduce(R, instances=2, protocol="LL128"), 16 << 20),
        ("ring_ch1_i16_LL128", P.ring_allreduce(R, instances=16, protocol="LL128"), 64 << 20),
        ("ring_ch1_i8_Simple", P.ring_allreduce(R, instances=8), 64 << 20),
        ("oneshot_Simple", P.oneshot_allreduce(R, protocol="Simple"), 4 << 20),
    ]
if SET == "ll128":
    cands = [
        ("ring_ch8_LL128", P.ring_allreduce(R, channels=8, protocol="LL128"), 64 << 20),
        ("ring_ch1_i16_LL128", P.ring_allreduce(R, instances=16, protocol="LL128"), 256 << 20),
        ("ring_ch1_i32_LL128", P.ring_allreduce(R, instances=32, protocol="LL128"), 256 << 20),
        ("ring_ch1_i8_Simple", P.ring_allreduce(R, instances=8), 256 << 20),
        ("ring_ch1_i32_Simple", P.ring_allreduce(R, instances=32), 256 << 20),
    ]
sizes = [1 << k for k in range(10, 31, 2)]
rows = {}
for name, algo, maxb in cands:
    progs = [c.load(algo.to_xml()) for c in comms]
    al = irparse.parse(algo.to_xml())
    for nbytes in sizes:
        if nbytes > maxb:
            continue
        n = nbytes // 2
        idx = torch.arange(n, device=dev)
        send = [synth.hashed(q, idx, "bfloat16") for q in range(R)]
        del idx
        recv = [torch.empty_like(x) for x in send]

        def call():
            with rt.group():
                for q in range(R):
                    comms[q].run(progs[q], send[q], recv[q], n)
        iters = 20 if nbytes <= (4 << 20) else 3
        t, mode = bench._timed(call, iters, stream, graph=nbytes <= (4 << 20))
        g = np.random.default_rng(3)
        smp = np.unique(np.concatenate([g.integers(0, n, 256), [0, n - 1]]))
        want = sampled.allreduce_at(al, lambda r, i: synth.hashed_numpy(r, i, "bfloat16"), n, "bfloat16", "sum", smp)
        got = recv[0][torch.from_numpy(smp).to(dev)].view(torch.int16).cpu().numpy().view(np.uint16)
        ok = bool(np.array_equal(got, want))
        bw = bench.busbw("allreduce", nbytes, t, R)
        rows.setdefault(nbytes, {})[name] = (t * 1e6, bw, ok)
        print(json.dumps({"program": name, "bytes": nbytes, "us": round(t * 1e6, 2), "busbw": round(bw, 2),
                          "mode": mode, "bit_exact": ok}), flush=True)
        del send, recv
        torch.cuda.empty_cache()
    for c, p in zip(comms, progs):
        c.unload(p)
names = [c[0] for c in cands]
lines = ["AllReduce bf16, 8 virtual ranks on one B200: time per call in us (busBW GB/s); * = bit-exact sampled parity",
         "", "| bytes/rank | " + " | ".join(names) + " | best |", "|---|" + "---|" * (len(names) + 1)]
for nb in sizes:
    r = rows.get(nb, {})
    cells = []
    for nm in names:
        if nm in r:
            us, bw, ok = r[nm]
            cells.append("%.1f (%.1f)%s" % (us, bw, "*" if ok else " MISMATCH"))
        else:
            cells.append("")
    best = min(r.items(), key=lambda kv: kv[1][0])[0] if r else ""
    lines.append("| %s | %s | %s |" % (nb, " | ".join(cells), best))
open(sys.argv[1] if len(sys.argv) > 1 else "/dev/stdout", "w").write("\n".join(lines) + "\n")
