"""Sweep for the 1-channel x k-instance virtual ring (slot size, slots, instances, threads)."""
import json, os, sys, argparse
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench

def run(**kw):
    ns = argparse.Namespace(gpus=1, steps=10, warmup=3, impl="msccl", ranks=8, size_mib=256.0, program="ring",
                            channels=1, instances=16, protocol="Simple", threads=512, slots=4, slot_kib=256,
                            no_e2e=True, no_cpu=True, quiet_extra=True)
    for k, v in kw.items():
        setattr(ns, k, v)
    try:
        r = bench.run_virtual(ns)
        bw = bench.busbw("allreduce", r["S"], r["t"], r["R"])
        print(json.dumps({**kw, "busbw": round(bw, 1), "ms": round(r["t"] * 1e3, 3), "bad": r["parity_bad"]}), flush=True)
    except Exception as e:
        print(json.dumps({**kw, "error": str(e)[:300]}), flush=True)

for inst in (8, 16, 18):
    run(instances=inst)
for sk, sl in [(64, 2), (64, 4), (128, 2), (128, 4), (512, 2), (512, 4), (1024, 2)]:
    run(slot_kib=sk, slots=sl)
for th in (256, 384):
    run(threads=th)
