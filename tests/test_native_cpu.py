"""CPU-side checks of the native library: it loads, exports every symbol include/msccl.h
declares, and its C++ validator agrees with the independent Python validator of the
oracle on valid programs and on every IR mutant (no compute calls: no GPU here)."""
import os
import re

import pytest

from oracle import irparse
from oracle import validate as pyval
from paper_conf_asplos_cowanmmsx23_b200 import programs as P

import irmutate

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def rt():
    from paper_conf_asplos_cowanmmsx23_b200 import runtime
    return runtime


def test_library_exports_every_declared_symbol(rt):
    hdr = open(os.path.join(ROOT, "include", "msccl.h")).read()
    names = set(re.findall(r"^(?:mscclResult_t|const char\*|uint64_t)\s+(msccl\w+)\(", hdr, re.M))
    assert len(names) >= 25
    for n in names:
        assert hasattr(rt.lib, n), n
    assert set(rt.SIGNATURES) == names


def test_error_strings_and_params(rt):
    assert rt.lib.mscclGetErrorString(8) == b"invalid MSCCL-IR program"
    assert rt.get_param("MSCCL_SLOTS") >= 1
    with pytest.raises(rt.MscclError):
        rt.set_param("NOPE", 1)


VALID = [
    ("ring4", lambda: P.ring_allreduce(4), 4),
    ("ring8ch", lambda: P.ring_allreduce(8, 8, 2), 8),
    ("allpairs8", lambda: P.allpairs_allreduce(8), 8),
    ("oneshot8", lambda: P.oneshot_allreduce(8), 8),
    ("hier", lambda: P.hierarchical_allreduce(2, 3), 6),
    ("ag", lambda: P.ring_allgather(4, 2, 2), 4),
    ("rs", lambda: P.ring_reducescatter(8, 2, 1), 8),
    ("a2a", lambda: P.alltoall_twostep(2, 4), 8),
    ("a2n", lambda: P.alltonext(2, 3), 6),
    ("nvls_ar", lambda: P.nvls_allreduce(8, 4), 8),
    ("nvls_rs", lambda: P.nvls_reducescatter(4, 2), 4),
    ("nvls_ag", lambda: P.nvls_allgather(8), 8),
]


@pytest.mark.parametrize("name,build,R", VALID, ids=[v[0] for v in VALID])
def test_cpp_validator_accepts_shipped_programs(rt, name, build, R):
    ok, msg = rt.validate(build().to_xml(), R, slots=2)
    assert ok, msg


@pytest.mark.parametrize("name,rule,text", irmutate.mutations(), ids=[m[0] for m in irmutate.mutations()])
def test_cpp_and_python_validators_agree_on_mutants(rt, name, rule, text):
    ok, msg = rt.validate(text, 4, slots=8)
    assert not ok
    assert msg.startswith(rule), msg
    with pytest.raises((pyval.ValidationError, irparse.IRError)) as ei:
        pyval.validate(irparse.parse(text), nranks=4, slots=8)
    assert str(ei.value)[:2] == msg[:2]


def test_cpp_deadlock_fixtures(rt):
    ring1 = P.ring_allreduce(4, inplace=True).to_xml()
    ok, msg = rt.validate(ring1, 4, slots=1)
    assert not ok and msg.startswith("V9")
    assert rt.validate(ring1, 4, slots=2)[0]
    assert rt.validate(P.ring_allreduce(8, channels=8, inplace=True).to_xml(), 8, slots=1)[0]
    ok, msg = rt.validate(irmutate.recv_before_send_ir(), 2, slots=8)
    assert not ok and msg.startswith("V9")
    text = irmutate.outstanding_sends_ir()
    assert not rt.validate(text, 2, slots=2)[0]
    assert rt.validate(text, 2, slots=3)[0]
    for K in (2, 3):  # K interleaved rings (reading R27) need K+1 slots, as in the oracle
        k = P.ring_allreduce(8, rings=K).to_xml()
        ok, msg = rt.validate(k, 8, slots=K)
        assert not ok and msg.startswith("V9")
        assert rt.validate(k, 8, slots=K + 1)[0]


def test_cpp_thread_block_limit(rt):
    over, text = irmutate.too_many_tbs(10)
    ok, msg = rt.validate(text, 8, max_tbs=10)
    assert not ok and msg.startswith("V4")


def test_cpp_parser_rejects_malformed(rt):
    for bad in ["", "<algo", "<gpu/>", '<algo name="x" coll="nope" ngpus="1" inplace="0"></algo>',
                '<algo name="x" coll="allreduce" ngpus="1" inplace="0"><gpu id="0" i_chunks="1" o_chunks="1">'
                '<tb id="0" send="-1" recv="-1" chan="0"><step s="0" type="zz" srcbuf="i" srcoff="0" dstbuf="o" '
                'dstoff="0" cnt="1" depid="-1" deps="-1" hasdep="0"/></tb></gpu></algo>']:
        ok, msg = rt.validate(bad, 1)
        assert not ok and msg.startswith("V1"), (bad, msg)


@pytest.mark.parametrize("seed", [0, 1, 2])
def test_cpp_and_python_validators_agree_on_random_mutants(rt, seed):
    """1000 seeded random IR mutants per seed: both validators accept, or both reject with
    the same rule (V1..V9)."""
    seen = set()
    accepted = 0
    for text, R in irmutate.random_mutants(seed, 1000):
        ok, msg = rt.validate(text, R, slots=8)
        try:
            pyval.validate(irparse.parse(text), nranks=R, slots=8)
            py = None
        except irparse.IRError:
            py = "V1"
        except pyval.ValidationError as e:
            py = str(e)[:2]
        cpp = None if ok else msg[:2]
        assert cpp == py, (cpp, msg, py, text)
        if cpp:
            seen.add(cpp)
        else:
            accepted += 1
    assert {"V1", "V2", "V3", "V4", "V5", "V6", "V7", "V8"} <= seen, seen  # V9: deadlock fixtures above
    assert 50 < accepted < 900


def test_cpp_v11_multimem_rules(rt):
    """V11 in the loader: multimem programs use the Simple protocol, never touch scratch, and
    hold their multimem ops in the same thread blocks on every rank (reading R23)."""
    ll = P.nvls_allreduce(4).to_xml().replace('proto="Simple"', 'proto="LL"')
    ok, msg = rt.validate(ll, 4)
    assert not ok and msg.startswith("V11"), msg
    sc = P.nvls_allreduce(4).to_xml().replace('type="mrs" srcbuf="i"', 'type="mrs" srcbuf="s"', 1).replace(
        's_chunks="0"', 's_chunks="4"')
    ok, msg = rt.validate(sc, 4)
    assert not ok and msg.startswith("V11"), msg
    from oracle import validate as pv
    for text in (ll, sc):
        with pytest.raises(pv.ValidationError, match="^V11"):
            pv.validate(irparse.parse(text), nranks=4)


def test_bench_probe_programs_are_valid(rt):
    """bench.py's latency probes (the empty program and the one-hop program) pass both
    validators and the race check."""
    import bench
    from oracle import races
    for R in (2, 8):
        for text in (bench.nop_ir(R), bench.hop_ir(R), bench.hop_ir(R, "LL128")):
            ok, msg = rt.validate(text, R)
            assert ok, msg
            al = irparse.parse(text)
            pyval.validate(al, nranks=R, races=True)
            assert races.find_races(al) == []


def test_direct_placement_needs_equal_chunk_lengths(rt):
    """A receive is placed directly only if the matching send's own destination chunk is as long
    as the receiver's for every count (same position in its block, or a scratch target), since a
    direct store stops at the receiver's chunk (reading R15; found by the random-program fuzzer).
    Here rank 0's rrcs writes its chunk 0 and forwards to rank 1's chunk 1 (the ragged one for
    counts that are not a multiple of the chunking): not direct; to rank 1's chunk 0: direct."""
    def prog(peer_off):
        return ('<algo name="len" coll="custom" ngpus="2" proto="Simple" inplace="0" nchannels="2" ninstances="1">'
                '<gpu id="0" i_chunks="2" o_chunks="2" s_chunks="0">'
                '<tb id="0" send="1" recv="1" chan="0"><step s="0" type="rrcs" srcbuf="i" srcoff="0" dstbuf="o" '
                'dstoff="0" cnt="1" depid="-1" deps="-1" hasdep="0"/></tb></gpu>'
                '<gpu id="1" i_chunks="2" o_chunks="2" s_chunks="0">'
                '<tb id="0" send="0" recv="-1" chan="0"><step s="0" type="s" srcbuf="i" srcoff="0" dstbuf="-" '
                'dstoff="-1" cnt="1" depid="-1" deps="-1" hasdep="0"/></tb>'
                '<tb id="1" send="-1" recv="0" chan="0"><step s="0" type="r" srcbuf="-" srcoff="-1" dstbuf="o" '
                'dstoff="%d" cnt="1" depid="-1" deps="-1" hasdep="0"/></tb></gpu></algo>' % peer_off)
    assert rt.validate(prog(1), 2)[0] and rt.validate(prog(0), 2)[0]
    assert rt.direct_placement(prog(1), 0)[0][0] & 3 == 0      # rank 0's rrcs: FIFO
    assert rt.direct_placement(prog(0), 0)[0][0] & 3 == 1      # same chunk position: direct
