"""GPU parity at production launch parameters (256 KiB slots, 256 threads, unrolled 256-bit
vector loops, L2 discard of consumed FIFO lines) with partial last tiles and ragged
chunks, plus sampled parity at the bench's full size (256 MiB per rank, 8 virtual ranks,
1 channel x 16 instances) against the oracle's reduction trees (oracle/sampled.py)."""
import numpy as np
import pytest

import synth
from oracle import irparse, sampled, sim
from paper_conf_asplos_cowanmmsx23_b200 import programs as P

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True, params=[1, 0], ids=["direct", "fifo"])
def production_params(request):
    """Production launch parameters; every test runs with direct placement (reading R15)
    and with it disabled (all messages through the receiver-side FIFO)."""
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    for k, v in (("MSCCL_SLOT_BYTES", 262144), ("MSCCL_LL_SLOT_BYTES", 65536), ("MSCCL_LL128_SLOT_BYTES", 262144),
                 ("MSCCL_SLOTS", 4), ("MSCCL_THREADS", 256), ("MSCCL_MAX_CHANNELS", 32), ("MSCCL_TIMEOUT_S", 10),
                 ("MSCCL_DIRECT", request.param)):
        runtime.set_param(k, v)
    yield
    runtime.set_param("MSCCL_DIRECT", 1)


@pytest.mark.parametrize("r,extra", [(4, 12345), (3, 7), (2, 131072 * 2 + 999)])
def test_ring_partial_tiles_default_slots(r, extra):
    import gpu_util
    R = 8
    n = R * r * 131072 * 2 + extra
    ir = P.ring_allreduce(R, instances=r).to_xml()
    xs = synth.inputs(R, n, "bfloat16", "uniform")
    want = sim.simulate(irparse.parse(ir), xs, n, "bfloat16", "sum")
    got = gpu_util.run_program(ir, xs, n, "bfloat16", "sum")
    for g, w in zip(got, want):
        assert np.array_equal(g, w)


def test_alltoall_and_allgather_default_slots():
    import gpu_util
    from oracle import mpi_ref
    R, n = 8, 300001
    xs = synth.inputs(R, R * n, "bfloat16", "pattern")
    got = gpu_util.run_program(P.alltoall_twostep(1, R, 1).to_xml(), xs, n, "bfloat16", out_elems=R * n)
    assert all(np.array_equal(g, e) for g, e in zip(got, mpi_ref.alltoall(xs, n)))
    xs = synth.inputs(R, n, "int32", "pattern")
    got = gpu_util.run_program(P.ring_allgather(R, 1, 4).to_xml(), xs, n, "int32", out_elems=R * n)
    assert all(np.array_equal(g, e) for g, e in zip(got, mpi_ref.allgather(xs)))


def test_protocols_share_connections():
    """Simple, LL128 and LL programs (and two tile sizes) alternate on the same connections
    of one communicator set: the monotone counters stay consistent across launches
    whatever protocol the previous launch used."""
    import gpu_util
    R = 8
    seq = [("Simple", 300001), ("LL128", 40000), ("Simple", 70001), ("LL", 9000), ("Simple", 300001),
           ("Simple", 5000), ("LL128", 300001), ("Simple", 131072 * 3 + 17)]
    for proto, n in seq:
        ir = P.ring_allreduce(R, instances=2, protocol=proto).to_xml()
        xs = synth.inputs(R, n, "float32", "uniform")
        want = sim.simulate(irparse.parse(ir), xs, n, "float32", "sum")
        got = gpu_util.run_program(ir, xs, n, "float32", "sum")
        for g, w in zip(got, want):
            assert np.array_equal(g.view(np.uint32), w.view(np.uint32)), (proto, n)


def test_mixed_protocols_small_int_payload_matching_sequence_numbers():
    """Simple, LL and LL128 programs alternate on one communicator set with int32
    data whose words equal the connections' upcoming message sequence numbers (1..400). A
    receiver that accepted stale bytes of another protocol as a valid LL / LL128 line (the
    flag check of an LL line is equality with the sequence number) would read old data. Each
    protocol has its own FIFO slots, so every result is bit-exact with the oracle."""
    import gpu_util
    R = 8
    seq = [("Simple", 60001), ("LL", 3001), ("Simple", 90001), ("LL128", 20001), ("LL", 5001), ("Simple", 40001),
           ("LL128", 7001), ("LL", 60001), ("Simple", 8001), ("LL", 12001)]
    for k, (proto, n) in enumerate(seq):
        ir = P.ring_allreduce(R, instances=2, protocol=proto).to_xml()
        xs = [((np.arange(n, dtype=np.int64) * (q + 3) + k) % 400 + 1).astype(np.int32) for q in range(R)]
        want = sim.simulate(irparse.parse(ir), xs, n, "int32", "max")
        got = gpu_util.run_program(ir, xs, n, "int32", "max")
        for g, w in zip(got, want):
            assert np.array_equal(g, w), (proto, n)


@pytest.mark.parametrize("instances", [16, 32])
def test_bench_size_sampled_parity(instances):
    """The bench workload (launch configuration of bench.py) at full size; outputs
    sampled on every rank and compared bit-exactly with the oracle's reduction trees."""
    import torch
    import gpu_util
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    R, n = 8, (256 << 20) // 2
    algo = P.ring_allreduce(R, instances=instances)
    ir = algo.to_xml()
    cs = gpu_util.comms(R)
    progs = [c.load(ir) for c in cs]
    try:
        dev = torch.device("cuda:0")
        idx = torch.arange(n, device=dev, dtype=torch.int64)
        send = [synth.hashed(q, idx, "bfloat16") for q in range(R)]
        del idx
        recv = [torch.empty(n, dtype=torch.bfloat16, device=dev) for _ in range(R)]
        for _ in range(2):
            with runtime.group():
                for q in range(R):
                    cs[q].allreduce(send[q], recv[q])
        torch.cuda.synchronize()
        al = irparse.parse(ir)
        g = np.random.default_rng(5)
        sample = np.unique(np.concatenate([g.integers(0, n, 2048), [0, n - 1]]))
        for q in range(R):
            want = sampled.allreduce_at(al, lambda rr, i: synth.hashed_numpy(rr, i, "bfloat16"), n, "bfloat16", "sum",
                                        sample, rank=q)
            got = recv[q][torch.from_numpy(sample).to(dev)].view(torch.int16).cpu().numpy().view(np.uint16)
            assert np.array_equal(got, want), "rank %d" % q
    finally:
        for c, p in zip(cs, progs):
            c.unload(p)


def test_bench_size_reducescatter_sampled_parity():
    """The bench's ReduceScatter extra (ring, 32 instances, 256 MiB input per rank) at full
    size; outputs sampled on every rank and compared bit-exactly with the oracle's reduction
    trees (oracle.sampled.reduction_at)."""
    import torch
    import gpu_util
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    R, n = 8, (256 << 20) // 2
    nb = n // R
    algo = P.ring_reducescatter(R, 1, 32)
    ir = algo.to_xml()
    cs = gpu_util.comms(R)
    progs = [c.load(ir) for c in cs]
    try:
        dev = torch.device("cuda:0")
        idx = torch.arange(n, device=dev, dtype=torch.int64)
        send = [synth.hashed(q, idx, "bfloat16") for q in range(R)]
        del idx
        recv = [torch.empty(nb, dtype=torch.bfloat16, device=dev) for _ in range(R)]
        with runtime.group():
            for q in range(R):
                cs[q].run(progs[q], send[q], recv[q], nb)
        torch.cuda.synchronize()
        al = irparse.parse(ir)
        g = np.random.default_rng(6)
        sample = np.unique(np.concatenate([g.integers(0, nb, 2048), [0, nb - 1]]))
        for q in range(R):
            want = sampled.reduction_at(al, lambda rr, i: synth.hashed_numpy(rr, i, "bfloat16"), nb, "bfloat16",
                                        "sum", sample, rank=q)
            got = recv[q][torch.from_numpy(sample).to(dev)].view(torch.int16).cpu().numpy().view(np.uint16)
            assert np.array_equal(got, want), "rank %d" % q
    finally:
        for c, p in zip(cs, progs):
            c.unload(p)


def test_more_than_2_pow_31_elements():
    """Maximum sizes: an int8 ring AllReduce of 2^31 + 12345 elements per rank (2 virtual
    ranks, 8 instances) -- element offsets beyond 32 bits in the chunk geometry (reading R1) and
    the data loops. int8 sums wrap, so every element is x0 + x1 mod 256 whatever the order; a
    million sampled elements and the whole ragged tail are checked."""
    import torch
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    n = (1 << 31) + 12345
    if torch.cuda.get_device_properties(0).total_memory < 6 * n:
        pytest.skip("needs 4 buffers of 2 GiB")
    g = torch.Generator(device="cuda").manual_seed(20230325)
    send = [torch.randint(-128, 128, (n,), dtype=torch.int8, device="cuda", generator=g) for _ in range(2)]
    recv = [torch.empty_like(s) for s in send]
    comms = runtime.Comm.virtual(2, 0)
    try:
        algo = P.ring_allreduce(2, instances=8)
        progs = [c.load(algo.to_xml()) for c in comms]
        with runtime.group():
            for c, p, s, r in zip(comms, progs, send, recv):
                c.run(p, s, r, n, dtype="int8")
        torch.cuda.synchronize()
        idx = torch.cat([torch.randint(0, n, (1 << 20,), device="cuda", generator=g),
                         torch.arange(n - 70000, n, device="cuda")])
        want = (send[0][idx].to(torch.int32) + send[1][idx].to(torch.int32)).to(torch.uint8).to(torch.int8)
        for r in recv:
            assert torch.equal(r[idx], want)
        for c, p in zip(comms, progs):
            c.unload(p)
    finally:
        for c in comms:
            c.destroy()


def test_allgather_output_beyond_4g_elements():
    """Maximum sizes: an AllGather of 2^31 + 777 uint8 elements per rank into a 2^32 + 1554
    element output (2 virtual ranks): block offsets b * n beyond 32 bits (reading R1); exact."""
    import torch
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    n = (1 << 31) + 777
    if torch.cuda.get_device_properties(0).total_memory < 8 * n:
        pytest.skip("needs 12 GiB")
    g = torch.Generator(device="cuda").manual_seed(7)
    send = [torch.randint(0, 256, (n,), dtype=torch.uint8, device="cuda", generator=g) for _ in range(2)]
    recv = [torch.empty(2 * n, dtype=torch.uint8, device="cuda") for _ in range(2)]
    comms = runtime.Comm.virtual(2, 0)
    try:
        algo = P.ring_allgather(2, 1, 4)
        progs = [c.load(algo.to_xml()) for c in comms]
        with runtime.group():
            for c, p, s, r in zip(comms, progs, send, recv):
                c.run(p, s, r, n, dtype="uint8")
        torch.cuda.synchronize()
        for r in recv:
            for q in range(2):
                assert torch.equal(r[q * n:(q + 1) * n], send[q])
        for c, p in zip(comms, progs):
            c.unload(p)
    finally:
        for c in comms:
            c.destroy()
