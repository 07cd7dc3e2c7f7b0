"""TMA variants (library chosen by MSCCL_LIB) x threads x instances."""
import json, os, sys, argparse
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import bench
from paper_conf_asplos_cowanmmsx23_b200 import runtime as rt

def run(tma=1, **kw):
    ns = argparse.Namespace(gpus=1, steps=10, warmup=3, impl="msccl", ranks=8, size_mib=256.0, program="ring",
                            channels=1, instances=18, protocol="Simple", threads=256, slots=4, slot_kib=256,
                            no_e2e=True, no_cpu=True, quiet_extra=True)
    for k, v in kw.items():
        setattr(ns, k, v)
    rt.set_param("MSCCL_TMA", tma)
    try:
        r = bench.run_virtual(ns)
        bw = bench.busbw("allreduce", r["S"], r["t"], r["R"])
        print(json.dumps({"lib": os.path.basename(rt.LIBPATH), "tma": tma, **kw, "busbw": round(bw, 1), "ms": round(r["t"] * 1e3, 3), "bad": r["parity_bad"]}), flush=True)
    except Exception as e:
        print(json.dumps({"lib": os.path.basename(rt.LIBPATH), "tma": tma, **kw, "error": str(e)[:200]}), flush=True)
        sys.exit(1)

for th, inst in [(256, 18), (512, 18), (256, 32), (256, 36), (128, 36), (128, 54)]:
    run(threads=th, instances=inst)
