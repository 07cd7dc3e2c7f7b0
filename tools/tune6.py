"""TMA data path sweep (virtual ring)."""
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
        print(json.dumps({"tma": tma, **kw, "busbw": round(bw, 1), "ms": round(r["t"] * 1e3, 3), "bad": r["parity_bad"]}), flush=True)
    except Exception as e:
        print(json.dumps({"tma": tma, **kw, "error": str(e)[:300]}), flush=True)

run(tma=0, threads=256, instances=32)
for th in (256, 512):
    for inst, sk in [(18, 256), (18, 512), (16, 256), (18, 128)]:
        run(threads=th, instances=inst, slot_kib=sk)
run(threads=512, instances=18, slot_kib=256, slots=2)
run(threads=128, instances=18, slot_kib=256)
