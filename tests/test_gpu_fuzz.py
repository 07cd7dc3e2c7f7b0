"""The interpreter on seeded random MSCCLang programs (tests/progfuzz.py): every written
output chunk bit-exact with the oracle simulator executing the same IR, under the Simple, LL
and LL128 protocols, with direct placement on and off (the loader's direct-placement analysis,
reading R15, meets programs nobody wrote by hand) and with the cross-launch protocol of the
multi-GPU deployment run in one launch (reading R28), for int32, bf16 and fp32 sums."""
import numpy as np
import pytest

import progfuzz
import synth
from oracle import irparse, sim

pytestmark = pytest.mark.gpu

PROTOS = ["Simple", "LL", "LL128"]
DTYPES = ["int32", "bfloat16", "float32"]


@pytest.fixture(scope="module")
def small_slots():
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    keys = ("MSCCL_SLOT_BYTES", "MSCCL_LL_SLOT_BYTES", "MSCCL_LL128_SLOT_BYTES", "MSCCL_TIMEOUT_S", "MSCCL_DIRECT",
            "MSCCL_CROSS_LAUNCH", "MSCCL_DIRECT_HINTS")
    old = {k: runtime.get_param(k) for k in keys}
    for k in keys[:3]:
        runtime.set_param(k, 4096)     # several tiles per chunk at these sizes
    runtime.set_param("MSCCL_TIMEOUT_S", 20)
    yield runtime
    for k, v in old.items():
        runtime.set_param(k, v)


@pytest.mark.parametrize("mode", ["direct", "nopull", "fifo", "cross"])
@pytest.mark.parametrize("block", range(6))
def test_random_programs_bit_exact_vs_oracle(small_slots, mode, block):
    """Modes: direct placement with pulled first hops (the default, readings R15 / R30), direct
    placement without pulls (MSCCL_DIRECT_HINTS 9), FIFO only, the cross-launch protocol."""
    import gpu_util
    runtime = small_slots
    runtime.set_param("MSCCL_DIRECT", 0 if mode == "fifo" else 1)
    runtime.set_param("MSCCL_CROSS_LAUNCH", 1 if mode == "cross" else 0)
    runtime.set_param("MSCCL_DIRECT_HINTS", 9 if mode == "nopull" else 25)
    direct = mode
    for seed in range(block * 50, (block + 1) * 50):
        proto = PROTOS[seed % 3]
        dtype = DTYPES[(seed // 3) % 3]
        prog = progfuzz.random_program(seed, protocol=proto)
        assert prog is not None
        algo, R, C, meaning = prog
        text = algo.to_xml()
        n = 16 * C * 37 * 2   # every (sub-)chunk a whole number of 16-byte vectors (reading R1)
        xs = synth.inputs(R, n, dtype, "int" if dtype == "int32" else "uniform", seed=seed)
        want = sim.simulate(irparse.parse(text), xs, n, dtype, "sum")
        # in-place programs run both in place and out of place (pre-copy, reading R8)
        got = gpu_util.run_program(text, xs, n, dtype, "sum", out_elems=n, inplace=algo.inplace and seed % 2 == 0)
        E = n // C
        for (r, _, k) in meaning:
            a = got[r][k * E:(k + 1) * E].view(np.uint8)
            b = want[r][k * E:(k + 1) * E].view(np.uint8)
            assert np.array_equal(a, b), (seed, proto, dtype, direct, r, k)


@pytest.mark.parametrize("op", ["max", "min", "prod"])
def test_random_programs_other_reductions(small_slots, op):
    """max / min / prod (reading R6; multimem has no product, so prod programs use LL / LL128
    or Simple without multimem rounds): written chunks bit-exact with the simulator."""
    import gpu_util
    runtime = small_slots
    runtime.set_param("MSCCL_DIRECT", 1)
    runtime.set_param("MSCCL_CROSS_LAUNCH", 0)
    for seed in range(2000, 2060):
        proto = PROTOS[seed % 3]
        dtype = DTYPES[(seed // 3) % 3]
        prog = progfuzz.random_program(seed, protocol=proto)
        assert prog is not None
        algo, R, C, meaning = prog
        text = algo.to_xml()
        if op == "prod" and ('type="mr' in text or 'type="ms' in text):
            continue
        n = 16 * C * 37 * 2
        dist = "int" if dtype == "int32" else "uniform"
        xs = synth.inputs(R, n, dtype, dist, seed=seed)
        want = sim.simulate(irparse.parse(text), xs, n, dtype, op)
        got = gpu_util.run_program(text, xs, n, dtype, op, out_elems=n, inplace=algo.inplace)
        E = n // C
        for (r, _, k) in meaning:
            a = got[r][k * E:(k + 1) * E].view(np.uint8)
            b = want[r][k * E:(k + 1) * E].view(np.uint8)
            assert np.array_equal(a, b), (seed, proto, dtype, op, r, k)


@pytest.mark.parametrize("mode", ["direct", "nopull", "fifo"])
def test_random_programs_ragged_sizes_whole_buffers(small_slots, mode):
    """Ragged counts (chunks of unequal length, reading R1 / R2; LL / LL128 partial lines): every
    output chunk the program writes, over its whole span, bit-exact with the simulator."""
    import random
    import gpu_util
    runtime = small_slots
    runtime.set_param("MSCCL_DIRECT", 0 if mode == "fifo" else 1)
    runtime.set_param("MSCCL_CROSS_LAUNCH", 0)
    runtime.set_param("MSCCL_DIRECT_HINTS", 9 if mode == "nopull" else 25)
    for seed in range(1000, 1100):
        proto = PROTOS[seed % 3]
        dtype = DTYPES[(seed // 3) % 3]
        prog = progfuzz.random_program(seed, protocol=proto)
        assert prog is not None
        algo, R, C, meaning = prog
        text = algo.to_xml()
        n = random.Random(seed).randint(1, 6000)
        xs = synth.inputs(R, n, dtype, "int" if dtype == "int32" else "uniform", seed=seed)
        want = sim.simulate(irparse.parse(text), xs, n, dtype, "sum")
        got = gpu_util.run_program(text, xs, n, dtype, "sum", out_elems=n, inplace=algo.inplace, fill=0)
        # Defined elements: the simulator models stale data (a chunk never written, the tail of a
        # longer chunk that received a shorter, ragged one, reading R2) as poison; running it again
        # with a different poison changes exactly the elements that depend on stale data. Every
        # element that does not must match bit for bit.
        want2 = _simulate_other_poison(text, xs, n, dtype)
        w = xs[0].itemsize
        checked = 0
        for r in range(R):
            wb = want[r].view(np.uint8).reshape(-1, w)
            w2 = want2[r].view(np.uint8).reshape(-1, w)
            gb = got[r].view(np.uint8).reshape(-1, w)
            defined = np.all(wb == w2, axis=1)
            checked += int(defined.sum())
            assert np.array_equal(gb[defined], wb[defined]), (seed, proto, dtype, mode, n, r)
        assert checked > 0 or not meaning


def _simulate_other_poison(text, xs, n, dtype):
    from oracle import numerics as nm
    orig = nm.poison

    def other(dt, m):   # finite, unlike the default NaN / int max
        if dt == "bfloat16":
            return np.full(m, 0x4049, dtype=np.uint16)
        if dt in ("float16", "float32", "float64"):
            return np.full(m, 3.25, dtype=nm.storage(dt))
        return np.full(m, -0x15A5A5A5, dtype=nm.storage(dt))   # negative: min against int max

    nm.poison = other
    try:
        return sim.simulate(irparse.parse(text), xs, n, dtype, "sum")
    finally:
        nm.poison = orig


def test_random_programs_with_one_fifo_slot(small_slots):
    """MSCCL_SLOTS=1: the programs V9 accepts with one slot (the loader re-checks at the launch's
    pipeline depth, reading R24) run to completion on the GPU -- the abstract machine's
    deadlock freedom holds for the interpreter -- and match the simulator; the ones it refuses
    are refused before anything is launched."""
    import gpu_util
    runtime = small_slots
    runtime.set_param("MSCCL_DIRECT", 1)
    runtime.set_param("MSCCL_CROSS_LAUNCH", 0)
    old = runtime.get_param("MSCCL_SLOTS")
    runtime.set_param("MSCCL_SLOTS", 1)
    ran = refused = 0
    try:
        for seed in range(3000, 3080):
            proto = PROTOS[seed % 3]
            prog = progfuzz.random_program(seed, protocol=proto)
            algo, R, C, meaning = prog
            text = algo.to_xml()
            n = 16 * C * 37 * 2
            xs = synth.inputs(R, n, "int32", "int", seed=seed)
            try:
                got = gpu_util.run_program(text, xs, n, "int32", "sum", out_elems=n, inplace=algo.inplace)
            except runtime.MscclError as e:
                assert e.code == 8 and "V9" in str(e), str(e)   # mscclInvalidProgram, deadlock
                refused += 1
                continue
            want = sim.simulate(irparse.parse(text), xs, n, "int32", "sum", slots=1)
            E = n // C
            for (r, _, k) in meaning:
                assert np.array_equal(got[r][k * E:(k + 1) * E], want[r][k * E:(k + 1) * E]), (seed, proto, r, k)
            ran += 1
    finally:
        runtime.set_param("MSCCL_SLOTS", old)
    assert ran > 0


@pytest.mark.parametrize("slot", [12544, 65536])
def test_random_programs_other_slot_sizes(small_slots, slot):
    """Other FIFO slot sizes (tile T and depth I follow, reading R3): written chunks bit-exact."""
    import gpu_util
    runtime = small_slots
    runtime.set_param("MSCCL_DIRECT", 1)
    runtime.set_param("MSCCL_CROSS_LAUNCH", 0)
    keys = ("MSCCL_SLOT_BYTES", "MSCCL_LL_SLOT_BYTES", "MSCCL_LL128_SLOT_BYTES")
    for k in keys:
        runtime.set_param(k, slot)
    try:
        for seed in range(4000, 4060):
            proto = PROTOS[seed % 3]
            dtype = DTYPES[(seed // 3) % 3]
            algo, R, C, meaning = progfuzz.random_program(seed, protocol=proto)
            text = algo.to_xml()
            n = 16 * C * 37 * 8
            xs = synth.inputs(R, n, dtype, "int" if dtype == "int32" else "uniform", seed=seed)
            want = sim.simulate(irparse.parse(text), xs, n, dtype, "sum")
            got = gpu_util.run_program(text, xs, n, dtype, "sum", out_elems=n, inplace=algo.inplace)
            E = n // C
            for (r, _, k) in meaning:
                assert np.array_equal(got[r][k * E:(k + 1) * E].view(np.uint8), want[r][k * E:(k + 1) * E].view(np.uint8)), \
                    (seed, proto, dtype, slot, r, k)
    finally:
        for k in keys:
            runtime.set_param(k, 4096)


def test_rrcs_direct_target_shorter_than_local_chunk(small_slots):
    """Fuzzer seed 10013 (Simple, bf16, 8206 elements: the last chunk is 38 elements): an rrcs
    whose matching receive lands in the ragged last chunk of the peer must not be a direct
    placement -- the direct store is cut to the receiver's chunk, which used to cut this rank's
    own stored result short as well. The loader now places such messages through the FIFO."""
    import gpu_util
    runtime = small_slots
    runtime.set_param("MSCCL_DIRECT", 1)
    runtime.set_param("MSCCL_CROSS_LAUNCH", 0)
    runtime.set_param("MSCCL_SLOT_BYTES", 8192)
    try:
        algo, R, C, meaning = progfuzz.random_program(10013, protocol="Simple")
        text = algo.to_xml()
        n = 8206
        xs = synth.inputs(R, n, "bfloat16", "uniform", seed=10013)
        got = gpu_util.run_program(text, xs, n, "bfloat16", "sum", out_elems=n, inplace=algo.inplace, fill=0)
        want = sim.simulate(irparse.parse(text), xs, n, "bfloat16", "sum")
        want2 = _simulate_other_poison(text, xs, n, "bfloat16")
        for r in range(R):
            a, b, g = (x.view(np.uint16) for x in (want[r], want2[r], got[r]))
            assert np.array_equal(g[a == b], a[a == b]), r
    finally:
        runtime.set_param("MSCCL_SLOT_BYTES", 4096)
