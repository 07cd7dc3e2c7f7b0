"""AllToAll (direct) tuning on virtual ranks: instances, slot size, threads."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, bench, synth
from paper_conf_asplos_cowanmmsx23_b200 import programs as P, runtime as rt
R = 8
S = 256 << 20
n = S // 2
dev = torch.device("cuda:0")
for th, sk, inst in [(256, 256, 1), (256, 256, 2), (512, 256, 1), (256, 512, 2), (128, 256, 4), (256, 128, 2)]:
    rt.set_param("MSCCL_THREADS", th)
    rt.set_param("MSCCL_SLOT_BYTES", sk * 1024)
    rt.set_param("MSCCL_MAX_CHANNELS", 32)
    comms = rt.Comm.virtual(R, 0)
    algo = P.alltoall_twostep(1, R, inst)
    progs = [c.load(algo.to_xml()) for c in comms]
    send = [synth.hashed(q, torch.arange(n, device=dev), "bfloat16") for q in range(R)]
    recv = [torch.empty_like(x) for x in send]
    def a2a():
        with rt.group():
            for q in range(R):
                comms[q].run(progs[q], send[q], recv[q], n // R)
    try:
        t, mode = bench._timed(a2a, 3, torch.cuda.current_stream(), graph=False)
        ok = all(torch.equal(recv[q].view(R, -1)[p], send[p].view(R, -1)[q]) for q in range(R) for p in range(R))
        print(json.dumps({"threads": th, "slot_kib": sk, "instances": inst, "busbw": round(bench.busbw("alltoall", S, t, R), 1),
                          "ms": round(t * 1e3, 3), "ok": ok}), flush=True)
    except Exception as e:
        print(json.dumps({"threads": th, "slot_kib": sk, "instances": inst, "error": str(e)[:200]}), flush=True)
    for c in comms:
        c.destroy()
    del send, recv
    torch.cuda.empty_cache()
