"""Fast GPU sanity check: a few programs vs the oracle with production params."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np
import synth
from oracle import irparse, sim, mpi_ref
from paper_conf_asplos_cowanmmsx23_b200 import programs as P, runtime
runtime.set_param("MSCCL_TIMEOUT_S", 5)
for k in ("MSCCL_THREADS", "MSCCL_SLOT_BYTES"):
    if os.environ.get(k):
        runtime.set_param(k, int(os.environ[k]))
import gpu_util

def case(name, algo, R, n, dtype="bfloat16", op="sum", dist="uniform"):
    ir = algo.to_xml()
    xs = synth.inputs(R, n, dtype, dist)
    want = sim.simulate(irparse.parse(ir), xs, n, dtype, op)
    got = gpu_util.run_program(ir, xs, n, dtype, op)
    bad = [q for q in range(R) if not np.array_equal(got[q].view(np.uint8), want[q].view(np.uint8))]
    print(name, "OK" if not bad else "FAIL ranks %s" % bad, flush=True)

case("ring8_LL128", P.ring_allreduce(8, protocol="LL128"), 8, 8 * 131072 * 3 + 17)
case("ring8_LL128_f32", P.ring_allreduce(8, instances=2, protocol="LL128"), 8, 300007, "float32")
case("allpairs_LL128", P.allpairs_allreduce(8, protocol="LL128"), 8, 100003)
case("ring8", P.ring_allreduce(8), 8, 8 * 131072 * 3 + 17)
case("ring8_inst4", P.ring_allreduce(8, instances=4), 8, 8 * 4 * 131072 * 2 + 1001)
case("ring4_f32", P.ring_allreduce(4), 4, 100003, "float32")
case("allpairs_simple", P.allpairs_allreduce(8, protocol="Simple"), 8, 200000)
case("hier", P.hierarchical_allreduce(2, 4), 8, 300001)
R, n = 8, 50001
xs = synth.inputs(R, R * n, "int32", "pattern")
got = gpu_util.run_program(P.alltoall_twostep(1, R).to_xml(), xs, n, "int32", out_elems=R * n)
print("a2a", "OK" if all(np.array_equal(g, e) for g, e in zip(got, mpi_ref.alltoall(xs, n))) else "FAIL", flush=True)
