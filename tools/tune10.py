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
        print(json.dumps({**kw, "busbw": round(bench.busbw("allreduce", r["S"], r["t"], r["R"]), 1), "ms": round(r["t"] * 1e3, 3), "bad": r["parity_bad"]}), flush=True)
    except Exception as e:
        print(json.dumps({**kw, "error": str(e)[:300]}), flush=True)
for th, inst, sk, sl in [(256, 32, 256, 4), (256, 32, 192, 4), (256, 24, 256, 4), (256, 40, 256, 4), (256, 32, 320, 4), (256, 36, 224, 4), (512, 16, 256, 4), (256, 28, 256, 4), (256, 32, 256, 4)]:
    run(threads=th, instances=inst, slot_kib=sk, slots=sl)
