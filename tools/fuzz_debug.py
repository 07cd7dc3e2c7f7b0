"""Debug helper: run one random program (tests/progfuzz.py) on the GPU and report, per written
output chunk, the first differing element against the oracle."""
import os, sys
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT); sys.path.insert(0, os.path.join(ROOT, "tests"))
import numpy as np
import progfuzz, synth, gpu_util
from oracle import irparse, sim
from paper_conf_asplos_cowanmmsx23_b200 import runtime

seed, proto, dtype = int(sys.argv[1]), sys.argv[2], sys.argv[3]
slot = int(sys.argv[4]) if len(sys.argv) > 4 else 4096
mult = int(sys.argv[5]) if len(sys.argv) > 5 else 3
for k in ("MSCCL_SLOT_BYTES", "MSCCL_LL_SLOT_BYTES", "MSCCL_LL128_SLOT_BYTES"):
    runtime.set_param(k, slot)
runtime.set_param("MSCCL_TIMEOUT_S", 20)
algo, R, C, meaning = progfuzz.random_program(seed, protocol=proto)
text = algo.to_xml()
n = 16 * C * 37 * mult
xs = synth.inputs(R, n, dtype, "int" if dtype == "int32" else "uniform", seed=seed)
want = sim.simulate(irparse.parse(text), xs, n, dtype, "sum")
got = gpu_util.run_program(text, xs, n, dtype, "sum", out_elems=n)
E = n // C
print("R", R, "C", C, "inst", algo.ninstances, "n", n, "E", E)
for (r, _, k) in sorted(meaning):
    a = got[r][k * E:(k + 1) * E]
    b = want[r][k * E:(k + 1) * E]
    bad = np.nonzero(a.view(np.uint8) != b.view(np.uint8))[0]
    print((r, k), "OK" if len(bad) == 0 else "BAD bytes %d..%d of %d (%d bad)" % (bad[0], bad[-1], a.nbytes, len(bad)))
