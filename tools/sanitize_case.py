"""Small cases for compute-sanitizer (memcheck / synccheck): every protocol, direct on/off, the
cross-launch protocol in one launch (MSCCL_CROSS_LAUNCH, reading R28), multimem programs, the
split-phase and K-ring schedules, ragged sizes."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np
import synth
from oracle import irparse, sim, mpi_ref
from paper_conf_asplos_cowanmmsx23_b200 import programs as P, runtime
runtime.set_param("MSCCL_TIMEOUT_S", 60)
runtime.set_param("MSCCL_SLOT_BYTES", 16384)
runtime.set_param("MSCCL_THREADS", 128)
import gpu_util
bad = 0
for cross, direct in ((0, 1), (0, 0), (1, 1)):
    runtime.set_param("MSCCL_DIRECT", direct)
    runtime.set_param("MSCCL_CROSS_LAUNCH", cross)
    direct = "%d%s" % (direct, "x" if cross else "")
    for name, algo, R, n, dt in [("ring", P.ring_allreduce(4, instances=2), 4, 20011, "bfloat16"),
                                 ("ring_LL", P.ring_allreduce(4, protocol="LL"), 4, 5001, "float32"),
                                 ("ring_split", P.ring_allreduce(4, channels=4, split_phases=True), 4, 9001, "bfloat16"),
                                 ("ring_k2", P.ring_allreduce(4, rings=2), 4, 9001, "float16"),
                                 ("ring_LL128", P.ring_allreduce(4, protocol="LL128"), 4, 5001, "float16"),
                                 ("allpairs", P.allpairs_allreduce(4, protocol="Simple"), 4, 3003, "float32"),
                                 ("oneshot", P.oneshot_allreduce(4), 4, 777, "int32"),
                                 ("hier", P.hierarchical_allreduce(2, 2), 4, 999, "float32"),
                                 ("nvls", P.nvls_allreduce(4, 2), 4, 4099, "bfloat16"),
                                 ("ring_mm", P.ring_rs_multimem_ag_allreduce(4, 2), 4, 3001, "float32")]:
        xs = synth.inputs(R, n, dt, "uniform" if dt != "int32" else "int")
        want = sim.simulate(irparse.parse(algo.to_xml()), xs, n, dt)
        got = gpu_util.run_program(algo.to_xml(), xs, n, dt)
        ok = all(np.array_equal(g.view(np.uint8), w.view(np.uint8)) for g, w in zip(got, want))
        bad += not ok
        print(direct, name, "OK" if ok else "FAIL", flush=True)
    R, n = 4, 1001
    xs = synth.inputs(R, R * n, "int8", "pattern")
    got = gpu_util.run_program(P.alltoall_twostep(2, 2).to_xml(), xs, n, "int8", out_elems=R * n)
    ok = all(np.array_equal(g, e) for g, e in zip(got, mpi_ref.alltoall(xs, n)))
    bad += not ok
    print(direct, "a2a", "OK" if ok else "FAIL", flush=True)
print("bad", bad)
