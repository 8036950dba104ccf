"""Pins for the oracle's sampler, threshold search (O4), partition (O3) and gap report (O6).

Sample -> Identify -> Extrapolate: PAPER L86-L90 (Fig. 2), uniform sampling L92, extrapolation by
identity L236; heavy iff w > t L272-L274; closest-prefix split Alg. 2 l.2-4 L216-L218.
"""
import json
import os

import numpy as np
import pytest

import oracle
import sginputs as gen

GOLD = os.path.join(os.path.dirname(__file__), "golden", "o4_worked_example.json")


def _cm(**kw):
    cm = oracle.CostModel()
    for k, v in kw.items():
        setattr(cm, k, v)
    return cm


def _golden():
    g = json.load(open(GOLD))
    cm = _cm(**g["cost_model"])
    rows = np.array(g["rows"], dtype=np.int64)
    return g, cm, rows[:, 0], rows[:, 1], rows[:, 2]


# ---- hash / sampler ---------------------------------------------------------------------------

def test_splitmix64_matches_numba_library():
    """The counter hash h(seed, tag, j) = sm(seed ^ sm(tag ^ sm(j))) (reading R4) pinned to an
    independent SplitMix64: numba's xoroshiro128+ seeding routine (Vigna's splitmix64.c)."""
    from numba.cuda.random import init_xoroshiro128p_state, xoroshiro128p_dtype
    st = np.zeros(1, dtype=xoroshiro128p_dtype)

    def sm(x):
        init_xoroshiro128p_state(st, 0, np.uint64(x))
        return int(st[0]["s0"])

    assert sm(0) == 0xE220A8397B1DCDAF  # first output of splitmix64 seeded with 0
    M = (1 << 64) - 1
    for seed, tag, j in [(0, 0, 0), (1, oracle.tag_sample(), 5), (123456789, 77, 2**40 + 3), (M, M, M)]:
        assert oracle.hash3(seed, tag, j) == sm(seed ^ sm(tag ^ sm(j)))


def test_sample_membership_definition_and_rate():
    n, seed, f = 200_000, 7, 0.05
    S = oracle.sample_rows(n, seed, f)
    assert np.all(np.diff(S) > 0)
    # rate within 4 sigma of Binomial(n, f)
    assert abs(len(S) - n * f) < 4 * np.sqrt(n * f * (1 - f))
    # membership matches the threshold comparison on a spot set (hash pinned above)
    Tf = int(f * 2**64)
    Sset = set(S.tolist())
    for i in range(0, n, 1013):
        assert (oracle.hash3(seed, oracle.tag_sample(), i) < Tf) == (i in Sset)
    assert len(oracle.sample_rows(n, seed, 1.0)) == n
    assert np.array_equal(oracle.sample_rows(n, seed, 1.0), np.arange(n))


def test_sample_rows_subrange_consistent():
    n, seed, f = 50_000, 3, 0.1
    full = oracle.sample_rows(n, seed, f)
    part = oracle.sample_rows(n, seed, f, 10_000, 30_000)
    assert np.array_equal(part, full[(full >= 10_000) & (full < 30_000)])


def test_horvitz_thompson_unbiased():
    """E[(n/|S|) * sum_{i in S} w_i] = W for a uniform sample (reading R3: whole rows, B intact)."""
    A = gen.config("rmat12")
    w = oracle.row_work(A, A)
    n, W = A.nrows, int(w.sum())
    est = []
    for seed in range(1000):
        S = oracle.sample_rows(n, seed, 0.02)
        est.append(n / max(len(S), 1) * w[S].sum())
    est = np.array(est)
    assert abs(est.mean() - W) < 3 * est.std(ddof=1) / np.sqrt(len(est))


# ---- O4 -----------------------------------------------------------------------------------------

def test_worked_example_costs_and_J():
    g, cm, w, a, u = _golden()
    for r in range(1, len(w)):
        assert oracle.cost_L(cm, w[r], a[r], u[r]) == g["c_L"][r]
        assert oracle.cost_H(cm, w[r], a[r], u[r]) == g["c_H"][r]
    for t, Jt in g["J"].items():
        assert oracle.J(cm, w, a, u, int(t)) == Jt
    thr, Jmin = oracle.threshold(cm, w, a, u)
    assert thr == g["thr_star"] and Jmin == g["J"][str(thr)]
    for t, r in g["r_percent"].items():
        assert oracle.heavy_share(w, int(t)) == pytest.approx(r, rel=1e-12)
    # the sample S = {r1, r3, r5}
    S = np.array(g["sample_rows"])
    for t, Jt in g["J_sample"].items():
        assert oracle.J(cm, w[S], a[S], u[S], int(t)) == Jt
    thr_s, _ = oracle.threshold(cm, w[S], a[S], u[S])
    assert thr_s == g["thr_s"]
    rep = oracle.gap_report(w, a, u, cm, thr_s)
    assert rep["thr_star"] == g["thr_star"]
    assert rep["dr_pp"] == pytest.approx(g["dr_pp"], rel=1e-12)
    assert rep["delta_rel"] == pytest.approx(g["delta_rel"], rel=1e-12)


def _rand_model(rng, capu):
    return _cm(kappa_L=int(rng.integers(0, 500)), lambda_L=int(rng.integers(1, 20)),
               sigma_L=int(rng.integers(0, 3)), rho_L=int(rng.integers(0, 30)),
               kappa_H=int(rng.integers(0, 5000)), lambda_H=int(rng.integers(1, 20)),
               tau_H=int(rng.integers(0, 10)), mu_H=int(rng.integers(0, 30)),
               tiles_fixed=int(rng.integers(1, 8)), capu=capu, cap_L=int(rng.integers(50, 400)))


@pytest.mark.parametrize("seed", range(12))
def test_sorted_argmin_equals_brute_force_over_every_integer_t(seed):
    """thr from the ascending-w sweep == argmin of the plain J(t) over EVERY integer t in
    [0, cap_L] (non-candidates included), smallest minimiser (reading R6)."""
    rng = np.random.default_rng(seed)
    n = int(rng.integers(1, 40))
    w = rng.integers(0, 300, n).astype(np.int64)
    w[rng.random(n) < 0.2] = 0
    if seed % 3 == 0:
        w[: n // 2] = w[0]  # ties on w
    a = np.where(w > 0, rng.integers(1, 30, n), 0).astype(np.int64)
    u = np.minimum(w, rng.integers(1, 300, n)).astype(np.int64)
    cm = _rand_model(rng, capu=int(rng.integers(0, 3)) * 16)
    Js = [oracle.J(cm, w, a, u, t) for t in range(0, cm.cap_L + 1)]
    best = min(Js)
    thr, Jmin = oracle.threshold(cm, w, a, u)
    assert Jmin == best
    assert thr == Js.index(best)


def test_full_sample_equals_exhaustive():
    """f = 1 => thr_s == thr* exactly (the sample is the input)."""
    A = gen.config("rmat10")
    cm = _cm(kappa_L=2000, lambda_L=40, sigma_L=0, rho_L=60, kappa_H=400000, lambda_H=25,
             tau_H=300, mu_H=30, tiles_fixed=1, capu=4096, cap_L=4096)
    s = oracle.sampled_threshold(A, A, 1.0, seed=5, cm=cm)
    thr_star, Jstar = oracle.exhaustive_threshold(A, A, cm)
    assert s.thr == thr_star and s.Jmin == Jstar


def test_heavy_share_monotone():
    A = gen.config("rmat11")
    w = oracle.row_work(A, A)
    ts = np.unique(np.concatenate([[0], w]))
    r = [oracle.heavy_share(w, int(t)) for t in ts[:: max(1, len(ts) // 200)]]
    assert all(x >= y for x, y in zip(r, r[1:]))
    assert oracle.heavy_share(w, 0) == 100.0 and oracle.heavy_share(w, int(w.max())) == 0.0


def test_empty_rows_cost_nothing_and_are_never_candidates():
    cm = _cm(kappa_L=5, lambda_L=1, kappa_H=7, lambda_H=1, tiles_fixed=1, cap_L=100)
    w = np.array([0, 0, 0], dtype=np.int64)
    a = np.zeros(3, dtype=np.int64)
    assert oracle.J(cm, w, a, a, 0) == 0
    assert oracle.threshold(cm, w, a, a) == (0, 0)


def test_candidates_clipped_to_cap():
    cm = _cm(kappa_L=0, lambda_L=1, kappa_H=10**6, lambda_H=1, tiles_fixed=1, cap_L=50)
    w = np.array([10, 40, 60, 90], dtype=np.int64)  # light always cheaper, but capped at 50
    one = np.ones(4, dtype=np.int64)
    thr, _ = oracle.threshold(cm, w, one, one)
    assert thr == 40


# ---- O3 -----------------------------------------------------------------------------------------

@pytest.mark.parametrize("G", [1, 2, 3, 4, 8])
def test_partition_properties(G):
    A = gen.config("rmat12")
    w = oracle.row_work(A, A)
    cuts = oracle.partition(w, G)
    n, W = len(w), int(w.sum())
    assert cuts[0] == 0 and cuts[-1] == n and np.all(np.diff(cuts) >= 0)
    P = np.concatenate([[0], np.cumsum(w)])
    for g in range(1, G):
        target = (W * g) // G
        j = cuts[g]
        # closest prefix: no boundary is strictly closer; ties -> smaller index
        d = np.abs(P - target)
        assert d[j] == d.min() and j == int(np.argmin(d))
    loads = np.array([P[cuts[g + 1]] - P[cuts[g]] for g in range(G)])
    assert np.all(np.abs(loads - W / G) <= w.max() + 1)


def test_partition_alg2_two_way_split_reading():
    """Alg. 2 with r% on the first part: cut where the inclusive prefix V_L[i] is closest to
    L_CPU = r L / 100 (G = 2, r = 50). Tiny hand case: w = [5, 1, 1, 1, 8] -> W = 16, target 8,
    prefixes 0,5,6,7,8,16 -> cut after row 3 (P[4] = 8)."""
    cuts = oracle.partition(np.array([5, 1, 1, 1, 8]), 2)
    assert list(cuts) == [0, 4, 5]
    # tie: w = [2, 2] target 2 -> P = 0,2,4 -> j = 1
    assert list(oracle.partition(np.array([2, 2]), 2)) == [0, 1, 2]
    # tie between two boundaries equally close: w = [1, 2, 1], W=4, target 2, P=0,1,3,4 -> |1-2|=|3-2| -> smaller j = 1
    assert list(oracle.partition(np.array([1, 2, 1]), 2)) == [0, 1, 3]


def test_partition_concatenation_equals_whole():
    """Concatenating the per-part row blocks of C equals C (rows are independent given B)."""
    A = gen.config("rmat10")
    w = oracle.row_work(A, A)
    cuts = oracle.partition(w, 4)
    whole = oracle.spgemm(A, A)
    cols, vals = [], []
    for g in range(4):
        R = oracle.spgemm(A, A, rows=np.arange(cuts[g], cuts[g + 1]))
        cols.append(R.col)
        vals.append(R.val)
    assert np.array_equal(np.concatenate(cols), whole.col)
    assert np.array_equal(np.concatenate(vals), whole.val)


# ---- the branches production uses: capu > 0 (non-exact u/capu), rho_L > 0 ----------------------

GOLD2 = os.path.join(os.path.dirname(__file__), "golden", "o4_capu_rho_example.json")


def test_worked_example_capu_and_rho_branches():
    """Hand-derived fixture (tests/golden/o4_capu_rho_example.json): R(u) = max(1, ceil(u/capu))
    at non-exact u/capu, and c_L's rho_L*u term.
    A floor instead of the ceil, or rho_L*(u+1), changes c_H / c_L of some row here."""
    g = json.load(open(GOLD2))
    cm = _cm(**g["cost_model"])
    rows = np.array(g["rows"], dtype=np.int64)
    w, a, u = rows[:, 0], rows[:, 1], rows[:, 2]
    for r in range(1, len(w)):
        assert oracle.cost_L(cm, w[r], a[r], u[r]) == g["c_L"][r]
        assert oracle.cost_H(cm, w[r], a[r], u[r]) == g["c_H"][r]
    for t, Jt in g["J"].items():
        assert oracle.J(cm, w, a, u, int(t)) == Jt
    thr, Jmin = oracle.threshold(cm, w, a, u)
    assert thr == g["thr_star"] and Jmin == g["J"][str(thr)]
    S = np.array(g["sample_rows"])
    for t, Jt in g["J_sample"].items():
        assert oracle.J(cm, w[S], a[S], u[S], int(t)) == Jt
    assert oracle.threshold(cm, w[S], a[S], u[S])[0] == g["thr_s"]


def test_worked_example_cost_split_nonexact_uh():
    """uh_i = min(w_i, ceil(w_i U_c / W_c)) at non-exact quotients (reading R19), capu > 0 and
    rho_L > 0 inside the per-row costs; closest-prefix cuts on their prefix."""
    g = json.load(open(GOLD2))
    cm = _cm(**g["cost_model"])
    sp = g["split"]
    wa = np.array(sp["rows_wa"], dtype=np.int64)
    w, a = wa[:, 0], wa[:, 1]
    costs = [oracle.row_cost(cm, sp["thr"], sp["comp"], int(x), int(y)) for x, y in zip(w, a)]
    assert costs == sp["cost"]
    for (wi, ai), uh, c in zip(sp["rows_wa"], sp["uh"], sp["cost"]):
        if wi == 0:
            continue
        ref = oracle.cost_L(cm, wi, ai, uh) if wi <= sp["thr"] else oracle.cost_H(cm, wi, ai, uh)
        assert ref == c
    for G, cuts in sp["cuts"].items():
        got, tot = oracle.partition_cost(cm, sp["thr"], sp["comp"], w, a, int(G))
        assert got.tolist() == cuts and tot == sp["total"]


def test_cost_H_tile_count_closed_form():
    """R(u) = max(1, tiles_fixed, ceil(u/capu)) for capu > 0 at every u in [0, 5*capu]: with every
    other constant 0 and tau_H = a = 1, c_H(u) IS R(u) (closed form, checked against integer ceil)."""
    for capu in (1, 3, 16, 100):
        for tf in (0, 1, 7):
            cm = _cm(tau_H=1, tiles_fixed=tf, capu=capu, cap_L=100)
            for uu in range(0, 5 * capu + 2):
                assert oracle.cost_H(cm, 0, 1, uu) == max(1, tf, -(-uu // capu))
    cm = _cm(tau_H=1, tiles_fixed=7, capu=0, cap_L=100)
    assert oracle.cost_H(cm, 0, 1, 12345) == 7


def test_cost_L_rho_term_closed_form():
    """With only rho_L = 1: c_L = u exactly; with only sigma_L = 1: u * ceil(log2 max(u, 2))."""
    cm = _cm(rho_L=1, cap_L=100)
    for uu in (0, 1, 2, 3, 17, 1000):
        assert oracle.cost_L(cm, 5, 1, uu) == uu
    cm = _cm(sigma_L=1, cap_L=100)
    for uu, lg in ((0, 1), (1, 1), (2, 1), (3, 2), (4, 2), (5, 3), (1024, 10), (1025, 11)):
        assert oracle.cost_L(cm, 5, 1, uu) == uu * lg


def test_cost_H_range_floor_tiles_fixed_with_capu():
    """R(u) = max(1, tiles_fixed, ceil(u/capu)) when capu > 0 (the heavy path's
    minimum number of column ranges for a row spanning all p columns is tiles_fixed). Hand values for
    tiles_fixed = 3, capu = 16: u = 4 -> 3, 40 -> 3 (2.5 -> 3), 48 -> 3, 49 -> 4 (3.06 -> 4), 150 -> 10."""
    cm = _cm(tau_H=1, tiles_fixed=3, capu=16, cap_L=100)
    for uu, R in ((0, 3), (4, 3), (40, 3), (48, 3), (49, 4), (150, 10)):
        assert oracle.cost_H(cm, 0, 1, uu) == R
    cm = _cm(kappa_H=100, lambda_H=1, tau_H=1, mu_H=1, tiles_fixed=3, capu=16, cap_L=100)
    # c_H(w=60, a=5, u=40) = 100 + 60 + 5*3 + 40 = 215 ; c_H(200, 10, 150) = 100 + 200 + 10*10 + 150 = 550
    assert oracle.cost_H(cm, 60, 5, 40) == 215 and oracle.cost_H(cm, 200, 10, 150) == 550
    # with tiles_fixed = 12 the floor dominates: c_H(200, 10, 150) = 100 + 200 + 10*12 + 150 = 570
    cm.tiles_fixed = 12
    assert oracle.cost_H(cm, 200, 10, 150) == 570
