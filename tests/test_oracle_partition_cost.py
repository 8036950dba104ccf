"""Pins for the oracle's cost-weighted partition (reading R19):
Alg. 2's closest-prefix split on the modeled per-row cost of O4 (L87-L89) instead
of the flops L_AB (L206) — the per-device "threshold vector" of L106."""
import json
import os

import numpy as np
import pytest

import oracle

GOLD = os.path.join(os.path.dirname(__file__), "golden", "o3_cost_partition_example.json")


def _cm(**kw):
    cm = oracle.CostModel()
    for k, v in kw.items():
        setattr(cm, k, v)
    return cm


def test_hand_examples():
    g = json.load(open(GOLD))
    cm = _cm(**g["cost_model"])
    for case in g["cases"]:
        wa = np.array(case["rows_wa"], dtype=np.int64)
        w, a = wa[:, 0], wa[:, 1]
        costs = [oracle.row_cost(cm, case["thr"], case["comp"], int(x), int(y)) for x, y in zip(w, a)]
        assert costs == case["cost"]
        for G, cuts in case["cuts"].items():
            got, tot = oracle.partition_cost(cm, case["thr"], case["comp"], w, a, int(G))
            assert got.tolist() == cuts and tot == case["total"]
        for G, cuts in case["flops_cuts"].items():
            assert oracle.partition(w, int(G)).tolist() == cuts


def test_estimated_u_enters_the_cost_models_exactly():
    """uh_i = min(w_i, ceil(w_i U_c / W_c)) plugged into c_L / c_H of O4, by class at thr."""
    g = json.load(open(GOLD))
    cm = _cm(**g["cost_model"])
    for case in g["cases"]:
        for (w, a), uh in zip(case["rows_wa"], case["uh"]):
            c = oracle.row_cost(cm, case["thr"], case["comp"], w, a)
            if w == 0:
                assert c == 0
            elif w <= case["thr"]:
                assert c == oracle.cost_L(cm, w, a, uh)
            else:
                assert c == oracle.cost_H(cm, w, a, uh)


@pytest.mark.parametrize("G", [1, 2, 3, 8])
def test_flops_model_reduces_to_work_partition(G):
    """lambda_L = lambda_H = 1 and every other constant 0: c_i = w_i, so the cuts are O3's."""
    rng = np.random.default_rng(G)
    w = rng.integers(0, 5000, size=997).astype(np.int64)
    w[rng.random(997) < 0.3] = 0
    a = rng.integers(1, 40, size=997).astype(np.int64)
    cm = _cm(lambda_L=1, lambda_H=1, cap_L=4096)
    comp = [rng.integers(1, 100), 100, rng.integers(1, 100), 100]
    for thr in (0, 100, 4096):
        cuts, tot = oracle.partition_cost(cm, thr, comp, w, a, G)
        assert cuts.tolist() == oracle.partition(w, G).tolist()
        assert tot == int(w.sum())


def test_no_compression_uses_w_as_u():
    cm = _cm(kappa_L=3, lambda_L=2, sigma_L=1, rho_L=5, kappa_H=7, lambda_H=1, tau_H=2, mu_H=3, tiles_fixed=1, capu=8,
             cap_L=4096)
    for w, a, thr in [(1, 1, 5), (7, 3, 5), (5000, 17, 4096), (64, 2, 10)]:
        c = oracle.row_cost(cm, thr, [10, 10, 10, 10], w, a)
        ref = oracle.cost_L(cm, w, a, w) if w <= thr else oracle.cost_H(cm, w, a, w)
        assert c == ref


@pytest.mark.parametrize("G", [2, 5, 8])
def test_part_loads_within_one_row_of_target(G):
    rng = np.random.default_rng(10 + G)
    w = (rng.pareto(1.2, size=3000) * 50).astype(np.int64)
    a = rng.integers(1, 30, size=3000).astype(np.int64)
    cm = _cm(kappa_L=100, lambda_L=8, kappa_H=10000, lambda_H=1, tau_H=60, mu_H=2, tiles_fixed=1, capu=4096, cap_L=4096)
    comp = [70, 100, 40, 100]
    thr = 300
    cuts, tot = oracle.partition_cost(cm, thr, comp, w, a, G)
    c = np.array([oracle.row_cost(cm, thr, comp, int(x), int(y)) for x, y in zip(w, a)])
    assert int(c.sum()) == tot
    assert cuts[0] == 0 and cuts[-1] == len(w) and np.all(np.diff(cuts) >= 0)
    P = np.concatenate([[0], np.cumsum(c)])
    for g in range(1, G):
        assert abs(int(P[cuts[g]]) - (tot * g) // G) <= int(c.max())
