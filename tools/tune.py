"""Sweep interpreter launch parameters for the virtual-rank ring AllReduce (one GPU)."""
import itertools, json, os, sys, argparse
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench

def run(**kw):
    a = bench.parse.__wrapped__() if hasattr(bench.parse, "__wrapped__") else None
    ns = argparse.Namespace(gpus=1, steps=10, warmup=3, impl="msccl", ranks=8, size_mib=256.0, program="ring",
                            channels=8, instances=2, protocol="Simple", threads=512, slots=4, slot_kib=256,
                            no_e2e=True, no_cpu=True, quiet_extra=True)
    for k, v in kw.items():
        setattr(ns, k, v)
    try:
        r = bench.run_virtual(ns)
        bw = bench.busbw("allreduce", r["S"], r["t"], r["R"])
        print(json.dumps({**kw, "busbw": round(bw, 1), "ms": round(r["t"] * 1e3, 3), "bad": r["parity_bad"]}), flush=True)
    except Exception as e:
        print(json.dumps({**kw, "error": str(e)[:200]}), flush=True)

grid = sys.argv[1] if len(sys.argv) > 1 else "basic"
if grid == "basic":
    for ch, inst in [(1, 8), (1, 16), (2, 4), (2, 8), (4, 2), (4, 4), (8, 1), (8, 2)]:
        run(channels=ch, instances=inst)
    for th in (256, 384):
        run(threads=th)
    for sk, sl in [(64, 4), (128, 4), (512, 4), (1024, 2), (256, 2), (256, 8)]:
        run(slot_kib=sk, slots=sl)
