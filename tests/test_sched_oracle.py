"""Pins for the scheduler oracle (oracle/sched.py) against the outcomes the
paper states in prose (tests/golden/sched_examples.json, each case citing its
passage) and against the invariants of Alg. 1/2."""
import json
import os

import numpy as np
import pytest

from oracle.sched import (MiccoSchedulerOracle, Pair, local_reuse_pattern, TWO_NEW, TWO_REPEATED_DIFF,
                          TWO_REPEATED_SAME, ONE_REPEATED)

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "sched_examples.json")


def _cases():
    with open(GOLDEN) as f:
        return json.load(f)["cases"]


@pytest.mark.parametrize("case", _cases(), ids=lambda c: c["name"])
def test_paper_examples(case):
    S = MiccoSchedulerOracle(case["num_gpu"], case["reuse_bd"], gpu_max_memory=1e30)
    for t, gs in case["resident"].items():
        S.res[int(t)] = set(gs)
    pairs = [Pair(a, b, 10_000 + i, 1.0, 1, 1, 1) for i, (a, b) in enumerate(case["pairs"])]
    got = S.run([pairs])[0]
    if "expected" in case:
        assert got == case["expected"]
    if "expected_counts" in case:
        assert [got.count(g) for g in range(case["num_gpu"])] == case["expected_counts"]


def test_fig4_patterns():
    """Fig. 4: A1,A2 on GPU0 → twoRepeatedSame; B1 on GPU0,
    B2 on GPU1 → twoRepeatedDiff; C1 on GPU0 → oneRepeated; D1,D2 → twoNew."""
    res = {1: {0}, 2: {0}, 3: {0}, 4: {1}, 5: {0}}
    assert local_reuse_pattern(res, 1, 2) == TWO_REPEATED_SAME
    assert local_reuse_pattern(res, 3, 4) == TWO_REPEATED_DIFF
    assert local_reuse_pattern(res, 5, 99) == ONE_REPEATED
    assert local_reuse_pattern(res, 98, 99) == TWO_NEW


def test_load_bound_invariant_random():
    """count[g] ≤ balanceNum + max(reuseBd) for every GPU and vector (L150),
    unless every GPU is full (the #14 fallback, impossible with ceil)."""
    rng = np.random.default_rng(0)
    for trial in range(50):
        ng = int(rng.integers(1, 9))
        bd = [int(x) for x in rng.integers(0, 3, size=3)]
        S = MiccoSchedulerOracle(ng, bd, gpu_max_memory=1e30)
        nxt = 1000
        for _ in range(5):
            n = int(rng.integers(1, 40))
            vec = []
            for _ in range(n):
                vec.append(Pair(int(rng.integers(0, 30)), int(rng.integers(0, 30)), nxt, 1.0, 1, 1, 1))
                nxt += 1
            got = S.run([vec])[0]
            bal = -(-n // ng)
            for g in range(ng):
                assert got.count(g) <= bal + max(bd)


def test_eviction_mode_prefers_free_memory():
    """Alg. 2 lines 12-17 (L199): once a candidate would be oversubscribed,
    the GPU with the most free memory is chosen even if it has more work."""
    S = MiccoSchedulerOracle(2, [0, 0, 0], gpu_max_memory=100)
    S.begin_vector(4)
    S.mem = [90, 10]
    S.com = [0.0, 5.0]
    p = Pair(1, 2, 3, 1.0, 5, 5, 5)
    assert S.assign(p, [0, 1]) == 1
    S.mem = [10, 10]
    assert S.assign(p, [0, 1]) == 0   # no oversubscription: least computation


def test_alg2_tie_breaks():
    """Alg. 2's ties: with no oversubscription, lines 7-10 take the least
    computation and, when several GPUs tie on it (GPUSelect.size() > 1), the least memory among
    them; under oversubscription, lines 12-16 take the least memory (the most capacity, Step-III
    L250) and break ties on it by the least computation.  Remaining ties go to the lowest id
    (reading #17 for the paper's random())."""
    S = MiccoSchedulerOracle(3, [0, 0, 0], gpu_max_memory=1000)
    S.begin_vector(3)
    p = Pair(1, 2, 3, 1.0, 5, 5, 5)
    S.com = [2.0, 2.0, 2.0]
    S.mem = [30, 10, 20]
    assert S.assign(p, [0, 1, 2]) == 1          # computation tied: least memory
    S.com = [2.0, 1.0, 2.0]
    assert S.assign(p, [0, 1, 2]) == 1          # least computation first
    S.com = [3.0, 3.0, 1.0]
    S.mem = [10, 10, 40]
    assert S.assign(p, [0, 1]) == 0             # full tie: lowest id
    # oversubscribed (GPU 2 would exceed the budget): least memory, ties by least computation
    S.mem = [50, 50, 990]
    S.com = [4.0, 1.0, 0.0]
    assert S.assign(p, [0, 1, 2]) == 1
    S.com = [1.0, 4.0, 0.0]
    assert S.assign(p, [0, 1, 2]) == 0
