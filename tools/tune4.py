"""More CTAs per SM: threads x instances sweep for the virtual ring (one GPU)."""
import json, os, sys, argparse
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench

def run(**kw):
    ns = argparse.Namespace(gpus=1, steps=10, warmup=3, impl="msccl", ranks=8, size_mib=256.0, program="ring",
                            channels=1, instances=16, protocol="Simple", threads=512, slots=4, slot_kib=512,
                            no_e2e=True, no_cpu=True, quiet_extra=True)
    for k, v in kw.items():
        setattr(ns, k, v)
    try:
        r = bench.run_virtual(ns)
        bw = bench.busbw("allreduce", r["S"], r["t"], r["R"])
        print(json.dumps({**kw, "busbw": round(bw, 1), "ms": round(r["t"] * 1e3, 3), "bad": r["parity_bad"]}), flush=True)
    except Exception as e:
        print(json.dumps({**kw, "error": str(e)[:300]}), flush=True)

for th, inst, sk in [(256, 32, 512), (256, 36, 512), (256, 32, 256), (256, 36, 256), (128, 64, 256), (128, 72, 256),
                     (256, 32, 128), (384, 18, 512), (512, 18, 512)]:
    run(threads=th, instances=inst, slot_kib=sk)
