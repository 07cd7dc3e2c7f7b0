"""Debug helper: run a program on virtual ranks under several parameter sets and report
where the output differs from the MPI definition (rank, element ranges)."""
import sys
import numpy as np
sys.path.insert(0, ".")
import synth
from oracle import mpi_ref
from paper_conf_asplos_cowanmmsx23_b200 import programs as P, runtime


def ranges(bad):
    idx = np.nonzero(bad)[0]
    if idx.size == 0:
        return []
    cuts = np.nonzero(np.diff(idx) > 1)[0]
    starts = np.concatenate([[idx[0]], idx[cuts + 1]])
    ends = np.concatenate([idx[cuts], [idx[-1]]])
    return list(zip(starts.tolist(), ends.tolist()))[:8]


def run(ir, xs, n, dtype, out_elems, want):
    import gpu_util
    got = gpu_util.run_program(ir, xs, n, dtype, out_elems=out_elems)
    res = []
    for q, (g, w) in enumerate(zip(got, want)):
        bad = g != w
        if bad.any():
            res.append((q, int(bad.sum()), ranges(bad)))
    return res


sys.path.insert(0, "tests")
R = 8
for direct in (0,):
    for warp in (0, 1):
        for n, inst in ((300001, 4), (300000, 4), (300001, 1), (1 << 18, 4), (65536 * 2 + 5, 1)):
            for k, v in (("MSCCL_SLOT_BYTES", 262144), ("MSCCL_SLOTS", 4), ("MSCCL_THREADS", 256),
                         ("MSCCL_MAX_CHANNELS", 32), ("MSCCL_TIMEOUT_S", 10), ("MSCCL_DIRECT", direct),
                         ("MSCCL_WARP_FLAGS", warp)):
                runtime.set_param(k, v)
            import gpu_util
            gpu_util._COMMS.clear()
            xs = synth.inputs(R, n, "int32", "pattern")
            r = run(P.ring_allgather(R, 1, inst).to_xml(), xs, n, "int32", R * n, mpi_ref.allgather(xs))
            print("allgather direct=%d warp=%d n=%d inst=%d:" % (direct, warp, n, inst), "OK" if not r else r, flush=True)
