"""Pins oracle/sampled.py (the per-element oracle the bench and the full-size GPU parity
tests use) to the simulator oracle/sim.py, which is itself pinned to the MPI collective
definitions and brute force (test_oracle_sim.py). Every output element of every rank is
evaluated through the reduction trees and compared bit-for-bit with a full simulation on
the same inputs, at ragged counts that leave a short last chunk."""
import numpy as np
import pytest

import synth
from oracle import irparse, sampled, sim
from paper_conf_asplos_cowanmmsx23_b200 import programs as P

pytestmark = pytest.mark.filterwarnings("ignore::RuntimeWarning")


def _inputs(R, n_in, dtype):
    return [synth.hashed_numpy(q, np.arange(n_in), dtype) for q in range(R)]


@pytest.mark.parametrize("dtype", ["bfloat16", "float32"])
@pytest.mark.parametrize("name,build", [
    ("ring", lambda R: P.ring_allreduce(R, 2, 2)),
    ("allpairs", lambda R: P.allpairs_allreduce(R)),
])
@pytest.mark.parametrize("n", [1000, 4099])
def test_allreduce_at_equals_simulation(name, build, dtype, n):
    R = 4
    al = irparse.parse(build(R).to_xml())
    xs = _inputs(R, n, dtype)
    want = sim.simulate(al, xs, n, dtype, "sum")
    idx = np.arange(n)
    for r in range(R):
        got = sampled.allreduce_at(al, lambda q, i: xs[q][i], n, dtype, "sum", idx, rank=r)
        assert np.array_equal(got, want[r]), "rank %d" % r


@pytest.mark.parametrize("dtype", ["bfloat16", "float32"])
@pytest.mark.parametrize("R,inst", [(4, 1), (4, 2), (8, 2)])
@pytest.mark.parametrize("n", [1000, 4099])
def test_reducescatter_at_equals_simulation(R, inst, dtype, n):
    al = irparse.parse(P.ring_reducescatter(R, 1, inst).to_xml())
    xs = _inputs(R, R * n, dtype)
    want = sim.simulate(al, xs, n, dtype, "sum")
    idx = np.arange(n)
    for r in range(R):
        got = sampled.reduction_at(al, lambda q, i: xs[q][i], n, dtype, "sum", idx, rank=r)
        assert np.array_equal(got, want[r][:n]), "rank %d" % r


def test_reduction_at_sensitive_to_rank_block():
    """A ReduceScatter output must come from the rank's own block of every input: reading
    block 0 for every rank (a plausible indexing slip) must fail."""
    R, n = 4, 512
    al = irparse.parse(P.ring_reducescatter(R, 1, 1).to_xml())
    xs = _inputs(R, R * n, "float32")
    r1 = sampled.reduction_at(al, lambda q, i: xs[q][i], n, "float32", "sum", np.arange(n), rank=1)
    r0 = sampled.reduction_at(al, lambda q, i: xs[q][i], n, "float32", "sum", np.arange(n), rank=0)
    assert not np.array_equal(r0, r1)
