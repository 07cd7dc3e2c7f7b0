"""The cross-launch protocol of the multi-GPU / one-process-per-GPU deployment, run with every
rank co-resident in ONE cooperative launch (MSCCL_CROSS_LAUNCH=1).

What the multi-GPU path adds over the virtual-rank path is device code, not data movement:
* system-scope fences and flags;
* per-connection launch ordinals and the receiver's ready line before the first direct store
  of a launch (reading R15b);
* the multimem group barrier with published buffer references (reading R23).
With MSCCL_CROSS_LAUNCH=1 the runtime takes exactly those branches (direct mode 2, multimem
mode 2, sysScope) although every rank is in the same grid. Because all ranks are co-resident,
no kernel waits on a kernel that might not be scheduled (B200_PROFILING.md: ranks that wait
on one another must not run as separate launches on one GPU). Every result is compared
bit-exactly with the oracle simulator, and the device counters prove that the cross-launch
handshakes and launches actually happened.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _algo(name, W, proto):
    from paper_conf_asplos_cowanmmsx23_b200 import programs as P
    return {
        "ring": lambda: P.ring_allreduce(W, protocol=proto),
        "ring_i2": lambda: P.ring_allreduce(W, instances=2, protocol=proto),
        "ring_ch": lambda: P.ring_allreduce(W, channels=W, protocol=proto),
        "ring_split": lambda: P.ring_allreduce(W, channels=W, split_phases=True, protocol=proto),
        "allpairs": lambda: P.allpairs_allreduce(W, protocol=proto),
        "oneshot": lambda: P.oneshot_allreduce(W, protocol=proto),
        "hier": lambda: P.hierarchical_allreduce(2, W // 2, protocol=proto),
        "a2a": lambda: P.alltoall_twostep(1, W, protocol=proto),
        "a2a_2step": lambda: P.alltoall_twostep(2, W // 2, protocol=proto),
        "allgather": lambda: P.ring_allgather(W, 1, 2, protocol=proto),
        "reducescatter": lambda: P.ring_reducescatter(W, 1, 2, protocol=proto),
        "nvls_ar": lambda: P.nvls_allreduce(W, 2),
        "nvls_rs": lambda: P.nvls_reducescatter(W, 2),
        "nvls_ag": lambda: P.nvls_allgather(W, 2),
        "ring_mm": lambda: P.ring_rs_multimem_ag_allreduce(W, 2),
    }[name]()


COLL = {"a2a": "alltoall", "a2a_2step": "alltoall", "allgather": "allgather", "nvls_ag": "allgather",
        "reducescatter": "reducescatter", "nvls_rs": "reducescatter"}

# (program, protocol, dtype, op, n per block)
CASES = [
    ("ring", "Simple", "float32", "sum", 20003),
    ("ring_i2", "Simple", "bfloat16", "sum", 30001),
    ("ring", "LL", "bfloat16", "sum", 3001),
    ("ring", "LL128", "float16", "sum", 9001),
    ("ring_ch", "Simple", "int32", "max", 12345),
    ("ring_split", "Simple", "bfloat16", "sum", 40009),
    ("allpairs", "Simple", "float32", "sum", 8191),
    ("allpairs", "LL", "float16", "sum", 2049),
    ("oneshot", "LL", "bfloat16", "sum", 512),
    ("oneshot", "Simple", "float32", "min", 4099),
    ("hier", "Simple", "float32", "sum", 16001),
    ("hier", "LL128", "int32", "sum", 5003),
    ("a2a", "Simple", "bfloat16", None, 6007),
    ("a2a_2step", "Simple", "int32", None, 2001),
    ("a2a", "LL", "int32", None, 777),
    ("allgather", "Simple", "int32", None, 7001),
    ("allgather", "LL128", "uint8", None, 3333),
    ("reducescatter", "Simple", "float32", "sum", 5001),
    ("reducescatter", "LL", "float32", "prod", 1201),
    ("nvls_ar", "Simple", "bfloat16", "sum", 20011),
    ("nvls_ar", "Simple", "int32", "max", 7001),
    ("nvls_rs", "Simple", "float32", "sum", 9001),
    ("nvls_ag", "Simple", "int32", None, 5003),
    ("ring_mm", "Simple", "float32", "sum", 12007),
]
# Simple programs with direct receives into in/out/scratch (the ready handshake fires)
DIRECT_EXPECTED = {"ring", "ring_i2", "ring_ch", "ring_split", "allpairs", "oneshot", "a2a", "a2a_2step", "allgather"}


@pytest.fixture(scope="module")
def cross_params():
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    keys = ("MSCCL_CROSS_LAUNCH", "MSCCL_SLOT_BYTES", "MSCCL_LL_SLOT_BYTES", "MSCCL_LL128_SLOT_BYTES",
            "MSCCL_TIMEOUT_S")
    old = {k: runtime.get_param(k) for k in keys}
    runtime.set_param("MSCCL_CROSS_LAUNCH", 1)
    runtime.set_param("MSCCL_SLOT_BYTES", 16384)   # several tiles per chunk at these sizes
    runtime.set_param("MSCCL_LL_SLOT_BYTES", 16384)
    runtime.set_param("MSCCL_LL128_SLOT_BYTES", 16384)
    runtime.set_param("MSCCL_TIMEOUT_S", 60)
    yield runtime
    for k, v in old.items():
        runtime.set_param(k, v)


def _inputs(name, W, n, dtype):
    import synth
    from oracle import geometry
    coll = COLL.get(name, "allreduce")
    dist = "pattern" if coll in ("alltoall", "allgather") or dtype == "uint8" else (
        "uniform" if dtype.startswith(("float", "bf")) else "int")
    return (synth.inputs(W, geometry.buffer_elems(coll, "i", W, n), dtype, dist),
            geometry.buffer_elems(coll, "o", W, n))


@pytest.mark.parametrize("W", [2, 4, 8])
@pytest.mark.parametrize("name,proto,dtype,op,n", CASES, ids=["%s-%s-%s" % (c[0], c[1], c[2]) for c in CASES])
def test_cross_launch_protocol_bit_exact(cross_params, W, name, proto, dtype, op, n):
    import torch
    from oracle import irparse, sim
    runtime = cross_params
    if name in ("hier", "a2a_2step") and W == 2:
        pytest.skip("needs 2 x G ranks with G >= 2")
    algo = _algo(name, W, proto)
    xs, out_elems = _inputs(name, W, n, dtype)
    want = sim.simulate(irparse.parse(algo.to_xml()), xs, n, dtype, op or "sum")
    comms = runtime.Comm.virtual(W, 0)
    try:
        progs = [c.load(algo.to_xml()) for c in comms]
        send = [torch.from_numpy(x.view(np.uint8).copy()).cuda() for x in xs]
        recv = [torch.full((out_elems * xs[0].itemsize,), 0xA5, dtype=torch.uint8, device="cuda") for _ in range(W)]
        s0 = [c.stats() for c in comms]
        for _ in range(2):   # twice: launch ordinals and ready lines of the second launch
            with runtime.group():
                for c, p, s, r in zip(comms, progs, send, recv):
                    c.run(p, s, r, n, op=op or "sum", dtype=dtype)
            torch.cuda.synchronize()
        for q in range(W):
            assert comms[q].async_error() == 0
            got = recv[q].cpu().numpy().view(xs[0].dtype)
            assert np.array_equal(got.view(np.uint8), want[q].view(np.uint8)), "rank %d differs from the oracle" % q
        s1 = [c.stats() for c in comms]
        d2 = sum(b["launches_direct2"] - a["launches_direct2"] for a, b in zip(s0, s1))
        hs = sum(b["cross_direct_handshakes"] - a["cross_direct_handshakes"] for a, b in zip(s0, s1))
        d1 = sum(b["launches_direct1"] - a["launches_direct1"] for a, b in zip(s0, s1))
        assert d1 == 0, "emulation must never take the one-launch direct mode"
        if proto == "Simple" and name in DIRECT_EXPECTED:
            assert d2 == 2 * W and hs > 0, (d2, hs)
        if proto != "Simple":
            assert hs == 0
        for c, p in zip(comms, progs):
            c.unload(p)
    finally:
        for c in comms:
            c.destroy()
