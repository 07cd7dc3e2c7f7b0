"""Debug helper: run one program on virtual ranks and print where GPU != oracle."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np
import synth
from oracle import irparse, sim
from paper_conf_asplos_cowanmmsx23_b200 import programs as P, runtime
runtime.set_param("MSCCL_SLOT_BYTES", int(os.environ.get("SLOT", 16384)))
runtime.set_param("MSCCL_TIMEOUT_S", 5)
import gpu_util

def case(name, algo, R, n, dtype="bfloat16", op="sum"):
    ir = algo.to_xml()
    xs = synth.inputs(R, n, dtype, "uniform")
    want = sim.simulate(irparse.parse(ir), xs, n, dtype, op)
    got = gpu_util.run_program(ir, xs, n, dtype, op)
    bad = False
    for q in range(R):
        d = np.nonzero(got[q].view(np.uint8).reshape(n, -1).any(axis=1) != False)  # placeholder
        diff = np.nonzero(got[q] != want[q])[0]
        if diff.size:
            bad = True
            print(name, "rank", q, "ndiff", diff.size, "first", diff[:5], "last", diff[-5:],
                  "got", got[q][diff[:3]], "want", want[q][diff[:3]])
    print(name, "OK" if not bad else "FAIL")

n = 3 * 8192 * 2 + 37
for proto in ("LL", "Simple"):
    case("allpairs_%s_R2" % proto, P.allpairs_allreduce(2, protocol=proto), 2, n)
    case("oneshot_%s_R2" % proto, P.oneshot_allreduce(2, protocol=proto), 2, n)
    case("allpairs_%s_R2_small" % proto, P.allpairs_allreduce(2, protocol=proto), 2, 1000)
print(P.allpairs_allreduce(2).to_xml())
