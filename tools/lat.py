"""Small-message latency sweep (virtual ranks, CUDA-graph replay)."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, bench, synth
from paper_conf_asplos_cowanmmsx23_b200 import programs as P, runtime as rt
R = 8
rt.set_param("MSCCL_THREADS", int(os.environ.get("THREADS", 256)))
comms = rt.Comm.virtual(R, 0)
dev = torch.device("cuda:0")
stream = torch.cuda.current_stream()
for name, algo in (("oneshot_LL", P.oneshot_allreduce(R, protocol="LL")),
                   ("allpairs_LL", P.allpairs_allreduce(R, protocol="LL")),
                   ("oneshot_Simple", P.oneshot_allreduce(R, protocol="Simple")),
                   ("ring_LL", P.ring_allreduce(R, protocol="LL")),
                   ("ring_ch8_LL", P.ring_allreduce(R, channels=8, protocol="LL"))):
    progs = [c.load(algo.to_xml()) for c in comms]
    row = {"program": name}
    for nbytes in (1024, 8192, 65536, 1 << 20, 4 << 20):
        n = nbytes // 2
        send = [synth.hashed(q, torch.arange(n, device=dev), "float16") for q in range(R)]
        recv = [torch.empty_like(x) for x in send]
        def call():
            with rt.group():
                for q in range(R):
                    comms[q].run(progs[q], send[q], recv[q], n)
        t, mode = bench._timed(call, 20, stream)
        row[str(nbytes)] = round(t * 1e6, 2)
        row["mode"] = mode
    print(json.dumps(row), flush=True)
    for c, p in zip(comms, progs):
        c.unload(p)
