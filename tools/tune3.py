"""Sweep slot / slice sizes for the sliced Simple protocol (virtual ring, one GPU)."""
import json, os, sys, argparse
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench
from paper_conf_asplos_cowanmmsx23_b200 import runtime as rt

def run(slice_kib=64, **kw):
    ns = argparse.Namespace(gpus=1, steps=10, warmup=3, impl="msccl", ranks=8, size_mib=256.0, program="ring",
                            channels=1, instances=16, protocol="Simple", threads=512, slots=4, slot_kib=512,
                            no_e2e=True, no_cpu=True, quiet_extra=True)
    for k, v in kw.items():
        setattr(ns, k, v)
    rt.set_param("MSCCL_SLICE_BYTES", slice_kib * 1024)
    try:
        r = bench.run_virtual(ns)
        bw = bench.busbw("allreduce", r["S"], r["t"], r["R"])
        print(json.dumps({"slice_kib": slice_kib, **kw, "busbw": round(bw, 1), "ms": round(r["t"] * 1e3, 3), "bad": r["parity_bad"]}), flush=True)
    except Exception as e:
        print(json.dumps({"slice_kib": slice_kib, **kw, "error": str(e)[:300]}), flush=True)

mode = sys.argv[1] if len(sys.argv) > 1 else "a"
if mode == "a":
    for sk, slk in [(512, 512), (512, 128), (512, 64), (512, 32), (256, 64), (256, 32), (128, 32), (128, 16), (64, 16), (1024, 64)]:
        run(slot_kib=sk, slice_kib=slk)
    for inst in (8, 18):
        run(instances=inst)
    run(threads=256)
