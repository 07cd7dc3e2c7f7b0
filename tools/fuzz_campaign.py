"""Long random-program campaign on the GPU (tests/progfuzz.py): seeds [lo, hi), each run under
a protocol / dtype / placement mode / slot size / count drawn from the seed, compared with the
oracle simulator on every element that does not depend on stale data (the simulator run with two
poisons, as in tests/test_gpu_fuzz.py). Prints one summary line and the failing seeds.

Usage: python tools/fuzz_campaign.py LO HI [MAX_N]   (needs a GPU; MAX_N = largest count, default 20000)
"""
import json
import os
import random
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))


def main():
    import numpy as np
    import gpu_util
    import progfuzz
    import synth
    from oracle import irparse, sim
    from oracle import numerics as nm
    from paper_conf_asplos_cowanmmsx23_b200 import runtime

    lo, hi = int(sys.argv[1]), int(sys.argv[2])
    max_n = int(sys.argv[3]) if len(sys.argv) > 3 else 20000
    runtime.set_param("MSCCL_TIMEOUT_S", 20)
    orig_poison = nm.poison

    def other(dt, m):   # finite, and for integers negative: min / max against the default
        if dt == "bfloat16":   # int max would ignore a large poison
            return np.full(m, 0x4049, dtype=np.uint16)
        if dt in ("float16", "float32", "float64"):
            return np.full(m, 3.25, dtype=nm.storage(dt))
        return np.full(m, -0x15A5A5A5, dtype=nm.storage(dt))

    stats = {"ran": 0, "refused_v9": 0, "fail": 0, "elements": 0}
    fails = []
    t0 = time.time()
    for seed in range(lo, hi):
        g = random.Random(seed * 7919 + 1)
        proto = g.choice(["Simple", "LL", "LL128"])
        dtype = g.choice(["int32", "bfloat16", "float32", "float16"])
        op = g.choice(["sum", "sum", "max", "min"])
        mode = g.choice(["direct", "fifo", "cross"])
        slot = g.choice([4096, 8192, 16384, 65536])
        slots = g.choice([2, 4, 4, 8])
        prog = progfuzz.random_program(seed, protocol=proto, max_ranks=8)
        if prog is None:
            fails.append((seed, "dsl refused"))
            continue
        algo, R, C, meaning = prog
        text = algo.to_xml()
        n = g.randint(1, max_n)
        for k in ("MSCCL_SLOT_BYTES", "MSCCL_LL_SLOT_BYTES", "MSCCL_LL128_SLOT_BYTES"):
            runtime.set_param(k, slot)
        runtime.set_param("MSCCL_SLOTS", slots)
        runtime.set_param("MSCCL_DIRECT", 0 if mode == "fifo" else 1)
        runtime.set_param("MSCCL_CROSS_LAUNCH", 1 if mode == "cross" else 0)
        if len(gpu_util._COMMS) > 6:   # bound the device memory held by cached communicator sets
            for cs in gpu_util._COMMS.values():
                for c in cs:
                    c.destroy()
            gpu_util._COMMS.clear()
        xs = synth.inputs(R, n, dtype, "int" if dtype == "int32" else "uniform", seed=seed)
        try:
            got = gpu_util.run_program(text, xs, n, dtype, op, out_elems=n, inplace=algo.inplace, fill=0)
        except runtime.MscclError as e:
            if e.code == 8 and "V9" in str(e):
                stats["refused_v9"] += 1
                continue
            fails.append((seed, "launch: %s" % str(e)[:120]))
            continue
        w1 = sim.simulate(irparse.parse(text), xs, n, dtype, op, slots=max(slots, 8))
        nm.poison = other
        try:
            w2 = sim.simulate(irparse.parse(text), xs, n, dtype, op, slots=max(slots, 8))
        finally:
            nm.poison = orig_poison
        w = xs[0].itemsize
        bad = 0
        for r in range(R):
            a = w1[r].view(np.uint8).reshape(-1, w)
            b = w2[r].view(np.uint8).reshape(-1, w)
            gb = got[r].view(np.uint8).reshape(-1, w)
            defined = np.all(a == b, axis=1)
            stats["elements"] += int(defined.sum())
            bad += int(np.count_nonzero(np.any(gb[defined] != a[defined], axis=1)))
        stats["ran"] += 1
        if bad:
            stats["fail"] += 1
            fails.append((seed, dict(proto=proto, dtype=dtype, op=op, mode=mode, slot=slot, slots=slots, n=n,
                                     bad=bad)))
    stats["seconds"] = round(time.time() - t0, 1)
    print(json.dumps({"seeds": [lo, hi], "max_n": max_n, **stats}))
    for f in fails[:40]:
        print("FAIL", f)


if __name__ == "__main__":
    main()
