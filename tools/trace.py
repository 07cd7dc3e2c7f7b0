"""Per-message phase breakdown of the Simple protocol (needs the MSCCL_TRACE build)."""
import ctypes, json, os, sys, argparse
os.environ.setdefault("MSCCL_TRACE", "1")
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import bench
from paper_conf_asplos_cowanmmsx23_b200 import runtime as rt
rt.lib.msccl_debug_trace.restype = ctypes.POINTER(ctypes.c_uint64)

def run(**kw):
    ns = argparse.Namespace(gpus=1, steps=5, warmup=2, impl="msccl", ranks=8, size_mib=256.0, program="ring",
                            channels=1, instances=32, protocol="Simple", threads=256, slots=4, slot_kib=256,
                            no_e2e=True, no_cpu=True, quiet_extra=True)
    for k, v in kw.items():
        setattr(ns, k, v)
    r = bench.run_virtual(ns)
    p = rt.lib.msccl_debug_trace()
    a = np.ctypeslib.as_array(p, shape=(4096, 8)).copy()
    n = int(a[:, 5].sum())
    tot = a[:, :5].sum(axis=0)
    names = ["wait_head", "barrier1", "data_t0", "barrier2", "post"]
    out = {k: round(float(v) / n / 1e3, 3) for k, v in zip(names, tot)}
    out.update(kw)
    out["msgs_per_cta_per_step"] = round(n / (ns.steps + ns.warmup + 1) / np.count_nonzero(a[:, 5]), 1)
    out["step_ms"] = round(r["t"] * 1e3, 3)
    print(json.dumps(out), flush=True)
    a[:] = 0
    np.ctypeslib.as_array(p, shape=(4096, 8))[:] = 0

if __name__ == "__main__":
    if len(sys.argv) > 1 and sys.argv[1] == "alltoall":
        for kib in (256, 1024):
            run(program="alltoall", instances=2, slot_kib=kib)
    else:
        for kib in (64, 128, 256, 512):
            run(slot_kib=kib)
