"""Per-vector reuse bounds: the vector features
the planner computes, the per-vector sweep, and the fitted regression (a random forest written
by tools/train_bounds.py into bounds_model.cpp) evaluated in C++ against scikit-learn's own
predictions on held-out vectors (tests/golden/bounds_model_check.json)."""
import json
import math
from pathlib import Path

import numpy as np
import pytest

import paper_conf_ipps_wangr0e22_b200 as M
from micco_inputs import workloads

from test_plan_replay import replay

GOLD = Path(__file__).resolve().parent / "golden" / "bounds_model_check.json"


def test_forest_matches_scikit_learn_on_heldout_vectors():
    g = json.loads(GOLD.read_text())
    assert len(g["features"]) >= 32
    for f, want in zip(g["features"], g["raw"]):
        raw, b = M.micco_predict_bounds(f)
        assert np.allclose(raw, want, rtol=0, atol=1e-9), (f, raw, want)
        for i in range(3):
            if abs(want[i] - math.floor(want[i]) - 0.5) > 1e-9:  # away from a rounding tie
                assert b[i] == min(2, max(0, math.floor(want[i] + 0.5)))


def _ctx(wl, **kw):
    kw.setdefault("mem_budget_bytes", 8 << 30)
    ctx = M.Context(dist_world=1, **kw)  # planning only: lazy nodes, no tensor data
    M.load_workload(ctx, wl)
    return ctx


def test_stage_features_and_modes():
    wl = workloads.c2_meson_set(n_graphs=400, N=64, Lt=16, rate=0.7, dist="gaussian", seed=11)
    ctx = _ctx(wl, window_graphs=32)
    for n in (2, 4):
        f, b, p_fixed = M.micco_plan_stages(ctx.h, n, "fixed", [1, 2, 0])
        assert np.all(b == [1, 2, 0])
        assert np.all(f[:, 4] == n) and np.all(f[:, 0] >= 1)
        assert np.all((f[:, 2] >= 0) & (f[:, 2] <= 1)) and np.all((f[:, 3] >= 0) & (f[:, 3] <= 1))
        assert np.all(f[:, 5] >= 0) and np.all(f[:, 1] > 10)  # operands are > 1 KiB
        assert f[0, 3] == 0.0  # nothing is resident before the first vector
        for mode in ("stage_sweep", "regression"):
            f2, b2, p2 = M.micco_plan_stages(ctx.h, n, mode)
            assert np.all((b2 >= 0) & (b2 <= 2)) and p2 > 0
            assert np.array_equal(f2[0], f[0])  # the first vector sees the same state
            again = M.micco_plan_stages(ctx.h, n, mode)
            assert np.array_equal(again[1], b2) and again[2] == p2  # deterministic
        # the per-vector sweep varies its choice with the vector
        _, bs, _ = M.micco_plan_stages(ctx.h, n, "stage_sweep")
        assert len(np.unique(bs, axis=0)) >= 1
    f1, b1, _ = M.micco_plan_stages(ctx.h, 1, "stage_sweep")  # one GPU: bounds are moot
    assert np.all(b1 == 0)
    ctx.close()


@pytest.mark.parametrize("mode", [1, 2])
def test_per_vector_bound_plans_replay(mode):
    wl = workloads.c2_meson_set(n_graphs=300, N=8, Lt=2, rate=0.7, dist="gaussian", flips=True, seed=5)
    budget = 1 << 30
    ctx = M.Context(mem_budget_bytes=budget, window_graphs=40, bound_model=mode)
    M.load_workload(ctx, wl)
    c = replay(ctx, 4, None, budget)  # reuse_bound NULL → options.bound_model
    assert c[5] > 0
