"""Debug helper: replay the fifo sequence of tests/test_gpu_large.py on shared comms and
report mismatch ranges of the AllGather after it."""
import sys
import numpy as np
sys.path.insert(0, ".")
sys.path.insert(0, "tests")
import synth
from oracle import irparse, mpi_ref, sim
from paper_conf_asplos_cowanmmsx23_b200 import programs as P, runtime
import gpu_util
from debug_warp import ranges  # noqa

warp = int(sys.argv[1])
for k, v in (("MSCCL_SLOT_BYTES", 262144), ("MSCCL_SLOTS", 4), ("MSCCL_THREADS", 256),
             ("MSCCL_MAX_CHANNELS", 32), ("MSCCL_TIMEOUT_S", 10), ("MSCCL_DIRECT", 0), ("MSCCL_WARP_FLAGS", warp)):
    runtime.set_param(k, v)
R = 8
seq = sys.argv[2].split(",")
for step in seq:
    if step.startswith("ring"):
        r, extra = {"ring4": (4, 12345), "ring3": (3, 7), "ring2": (2, 131072 * 2 + 999)}[step]
        n = R * r * 131072 * 2 + extra
        ir = P.ring_allreduce(R, instances=r).to_xml()
        xs = synth.inputs(R, n, "bfloat16", "uniform")
        want = sim.simulate(irparse.parse(ir), xs, n, "bfloat16", "sum")
        got = gpu_util.run_program(ir, xs, n, "bfloat16", "sum")
    elif step == "a2a":
        n = 300001
        xs = synth.inputs(R, R * n, "bfloat16", "pattern")
        got = gpu_util.run_program(P.alltoall_twostep(1, R, 1).to_xml(), xs, n, "bfloat16", out_elems=R * n)
        want = mpi_ref.alltoall(xs, n)
    elif step == "ag":
        n = 300001
        xs = synth.inputs(R, n, "int32", "pattern")
        got = gpu_util.run_program(P.ring_allgather(R, 1, 4).to_xml(), xs, n, "int32", out_elems=R * n)
        want = mpi_ref.allgather(xs)
    res = []
    for q, (g, w) in enumerate(zip(got, want)):
        bad = g.view(np.uint8) != w.view(np.uint8)
        if bad.any():
            res.append((q, int(bad.sum()), ranges(bad)))
    print("warp=%d %s:" % (warp, step), "OK" if not res else res[:3], flush=True)
