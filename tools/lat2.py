"""Latency floor and small-message latency (virtual ranks, CUDA-graph replay)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, bench, synth
from paper_conf_asplos_cowanmmsx23_b200 import programs as P, runtime as rt
from paper_conf_asplos_cowanmmsx23_b200.dsl import Program, AllReduce, chunk
R = 8
rt.set_param("MSCCL_THREADS", int(os.environ.get("THREADS", 256)))
comms = rt.Comm.virtual(R, 0)
dev = torch.device("cuda:0")
stream = torch.cuda.current_stream()
with Program("localcopy", AllReduce(R, 1), protocol="LL") as p:
    for r in range(R):
        chunk(r, "in", 0).copy(r, "out", 0)
floor = p.lower()
with Program("pingring", AllReduce(R, 1), protocol="LL") as p:   # one hop per rank
    for r in range(R):
        chunk(r, "in", 0).copy((r + 1) % R, "out", 0)
hop = p.lower()
for name, algo in (("floor_localcopy", floor), ("one_hop_LL", hop),
                   ("oneshot_LL", P.oneshot_allreduce(R, protocol="LL")),
                   ("allpairs_LL", P.allpairs_allreduce(R, protocol="LL")),
                   ("ring_ch8_LL", P.ring_allreduce(R, channels=8, protocol="LL")),
                   ("ring_ch8_LL128", P.ring_allreduce(R, channels=8, protocol="LL128")),
                   ("allpairs_LL128", P.allpairs_allreduce(R, protocol="LL128"))):
    progs = [c.load(algo.to_xml()) for c in comms]
    row = {"program": name, "ctas": sum(pp.info()["thread_blocks"] for pp in progs)}
    for nbytes in (1024, 65536, 1 << 20):
        n = nbytes // 2
        send = [synth.hashed(q, torch.arange(n, device=dev), "float16") for q in range(R)]
        recv = [torch.empty_like(x) for x in send]
        def call():
            with rt.group():
                for q in range(R):
                    comms[q].run(progs[q], send[q], recv[q], n)
        t, mode = bench._timed(call, 20, stream)
        row[str(nbytes)] = round(t * 1e6, 2)
    print(json.dumps(row), flush=True)
    for c, pp in zip(comms, progs):
        c.unload(pp)
