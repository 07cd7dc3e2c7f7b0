"""Candidate programs at chosen sizes on 8 virtual ranks (CUDA-graph replay, 20 warm-up + 50
timed, bit-exact sampled parity of the last call): the data behind the size ranges of
programs.tuned_allreduce. Usage: python tools/candidates.py [out.jsonl]"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import bench  # noqa: E402
import synth  # noqa: E402
from paper_conf_asplos_cowanmmsx23_b200 import programs as P  # noqa: E402
from paper_conf_asplos_cowanmmsx23_b200 import runtime as rt  # noqa: E402

W = 8
rt.set_param("MSCCL_MAX_CHANNELS", 64)
comms = rt.Comm.virtual(W, 0)
R = bench.Ranks(rt, comms, list(range(W)), W, 1, torch.device("cuda:0"))
stream = torch.cuda.current_stream()
CANDS = [
    ("oneshot_LL", P.oneshot_allreduce(W, protocol="LL"), 64 << 10),
    ("allpairs_LL", P.allpairs_allreduce(W, protocol="LL"), 1 << 20),
    ("ring_ch8_LL", P.ring_allreduce(W, channels=8, protocol="LL"), 2 << 20),
    ("ring_ch8_LL128", P.ring_allreduce(W, channels=8, protocol="LL128"), 16 << 20),
    ("ring_ch8_i2_LL128", P.ring_allreduce(W, channels=8, instances=2, protocol="LL128"), 16 << 20),
    ("allpairs_i2_Simple", P.allpairs_allreduce(W, instances=2, protocol="Simple"), 16 << 20),
    ("ring_i8_Simple", P.ring_allreduce(W, instances=8), 64 << 20),
    ("ring_i32_Simple", P.ring_allreduce(W, instances=32), 64 << 20),
]
SIZES = [1 << k for k in range(10, 25)]
out = open(sys.argv[1], "w") if len(sys.argv) > 1 else None
for name, algo, maxb in CANDS:
    progs = R.load(algo)
    for size in SIZES:
        if size > maxb:
            continue
        n = size // 2
        send = [synth.hashed(q, torch.arange(n, device=R.dev), "bfloat16") for q in range(W)]
        recv = [torch.empty_like(x) for x in send]
        t, mode = bench.timed(lambda: R.call(progs, send, recv, n), 50, 20, stream, True, R)
        bad, _ = bench.sampled_parity(algo, recv, n, [0, W - 1])
        rec = {"program": name, "bytes": size, "us": round(t * 1e6, 2), "busbw": round(bench.busbw("allreduce", size, t, W), 2),
               "mode": mode, "correct": bad == 0}
        print(json.dumps(rec), flush=True)
        if out:
            out.write(json.dumps(rec) + "\n")
        del send, recv
    R.unload(progs)
