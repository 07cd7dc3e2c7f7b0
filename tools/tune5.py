"""Slots x slot-size at 2 CTAs/SM (virtual ring)."""
import json, os, sys, argparse
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench

def run(**kw):
    ns = argparse.Namespace(gpus=1, steps=10, warmup=3, impl="msccl", ranks=8, size_mib=256.0, program="ring",
                            channels=1, instances=32, protocol="Simple", threads=256, slots=4, slot_kib=256,
                            no_e2e=True, no_cpu=True, quiet_extra=True)
    for k, v in kw.items():
        setattr(ns, k, v)
    try:
        r = bench.run_virtual(ns)
        bw = bench.busbw("allreduce", r["S"], r["t"], r["R"])
        print(json.dumps({**kw, "busbw": round(bw, 1), "ms": round(r["t"] * 1e3, 3), "bad": r["parity_bad"]}), flush=True)
    except Exception as e:
        print(json.dumps({**kw, "error": str(e)[:300]}), flush=True)

for sl, sk in [(2, 128), (2, 192), (2, 256), (3, 192), (3, 256), (8, 256), (2, 384), (4, 384)]:
    run(slots=sl, slot_kib=sk)
run(threads=128, instances=64, slots=2, slot_kib=192)
run(threads=192, instances=36, slots=2, slot_kib=256)
