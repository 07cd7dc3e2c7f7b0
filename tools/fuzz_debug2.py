"""Debug helper: one random program at a ragged size, whole buffers (zero-filled) GPU vs oracle."""
import os, sys, random
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np
import progfuzz, synth, gpu_util
from oracle import irparse, sim
from paper_conf_asplos_cowanmmsx23_b200 import runtime

seed, proto, dtype = int(sys.argv[1]), sys.argv[2], sys.argv[3]
n = int(sys.argv[4]) if len(sys.argv) > 4 else random.Random(seed).randint(1, 6000)
for k in ("MSCCL_SLOT_BYTES", "MSCCL_LL_SLOT_BYTES", "MSCCL_LL128_SLOT_BYTES"):
    runtime.set_param(k, 4096)
runtime.set_param("MSCCL_TIMEOUT_S", 20)
algo, R, C, meaning = progfuzz.random_program(seed, protocol=proto)
text = algo.to_xml()
xs = synth.inputs(R, n, dtype, "int" if dtype == "int32" else "uniform", seed=seed)
want = sim.simulate(irparse.parse(text), xs, n, dtype, "sum")
got = gpu_util.run_program(text, xs, n, dtype, "sum", out_elems=n, inplace=algo.inplace, fill=0)
print("R", R, "C", C, "inst", algo.ninstances, "inplace", algo.inplace, "n", n)
for r in range(R):
    bad = np.nonzero(got[r] != want[r])[0]
    print(r, "OK" if len(bad) == 0 else "BAD elems %d..%d (%d): got %s want %s" % (bad[0], bad[-1], len(bad), got[r][bad[:4]], want[r][bad[:4]]))
if len(sys.argv) > 5:
    print(text)
