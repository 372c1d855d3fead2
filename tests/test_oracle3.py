"""Pins of the third-order oracle (oracle.search3 / tables3) against things other
than itself: the 4-way oracle tables marginalised over the fourth SNP (a separately written per-sample loop),
a closed form, and an independent numpy K2 over all triples of a tiny dataset."""
import itertools
import math

import numpy as np

import datagen
import oracle


def _k2_numpy(t):
    r0, r1 = t[0].astype(np.int64), t[1].astype(np.int64)
    return sum(math.lgamma(a + b + 2) - math.lgamma(a + 1) - math.lgamma(b + 1) for a, b in zip(r0, r1))


def test_triple_tables_are_quad_marginals():
    d = datagen.make_config("C1")
    rng = np.random.default_rng(3)
    for _ in range(20):
        i, j, k, l = sorted(rng.choice(d.n_snps, 4, replace=False))
        t3 = oracle.tables3(d.geno, d.phen, [[i, j, k]])[0]
        q = oracle.tables(d.geno, d.phen, [[i, j, k, l]])[0].reshape(2, 27, 3).sum(axis=2)
        np.testing.assert_array_equal(t3, q)
        assert t3[0].sum() == d.n_controls and t3[1].sum() == d.n_cases


def test_triple_k2_closed_form_identical_samples():
    geno = np.zeros((3, 40), dtype=np.uint8)
    phen = np.array([0] * 15 + [1] * 25, dtype=np.uint8)
    idx, k2 = oracle.search3(geno, phen, top_k=1)
    want = math.lgamma(40 + 2) - math.lgamma(15 + 1) - math.lgamma(25 + 1)
    assert abs(k2[0] - want) < 1e-9 * want and int(idx[0]) == oracle.pack_index(0, 1, 2, 0)


def test_triple_search_equals_numpy_brute_force():
    d = datagen.make_dataset(12, 30, 34, 99, planted=None, name="tiny3")
    tri = list(itertools.combinations(range(12), 3))
    tabs = oracle.tables3(d.geno, d.phen, tri)
    keys = sorted((_k2_numpy(t), oracle.pack_index(i, j, k, 0)) for t, (i, j, k) in zip(tabs, tri))
    idx, k2 = oracle.search3(d.geno, d.phen, top_k=10)
    assert [int(v) for v in idx] == [kk[1] for kk in keys[:10]]
    np.testing.assert_allclose(k2, [kk[0] for kk in keys[:10]], rtol=1e-12)


# ---- mutual-information objective ----------------------------------------------
def _mi_numpy(t):
    """M * I from the definition sum p(g, y) ln(p(g, y) / (p(g) p(y))), numpy, cells with r > 0 only."""
    t = t.astype(np.float64)
    M = t.sum()
    pg = t.sum(axis=0) / M
    py = t.sum(axis=1) / M
    s = 0.0
    for p in range(2):
        for c in range(t.shape[1]):
            if t[p, c] > 0:
                pj = t[p, c] / M
                s += pj * math.log(pj / (pg[c] * py[p]))
    return M * s


def test_mi_matches_definition_and_closed_forms():
    d = datagen.make_config("C1")
    tabs = oracle.tables(d.geno, d.phen, [[0, 1, 2, 3], [3, 11, 22, 35], [5, 9, 17, 30]])
    for t in tabs:
        assert abs(oracle.mi(t) - _mi_numpy(t)) < 1e-9 * max(1.0, abs(_mi_numpy(t)))
    # independence: every cell split in the class ratio -> MI = 0; perfect association -> M * H(phenotype)
    ind = np.zeros((2, 81), dtype=np.uint32)
    ind[0, :10], ind[1, :10] = 3, 1
    assert abs(oracle.mi(ind)) < 1e-9
    perf = np.zeros((2, 81), dtype=np.uint32)
    perf[0, 0], perf[1, 80] = 30, 10
    want = -(30 * math.log(30 / 40) + 10 * math.log(10 / 40))
    assert abs(oracle.mi(perf) - want) < 1e-9 * want


def test_mi_search_equals_numpy_ranking():
    d = datagen.make_dataset(9, 20, 24, 5, planted=None, name="tinymi")
    quads = list(itertools.combinations(range(9), 4))
    tabs = oracle.tables(d.geno, d.phen, quads)
    keys = sorted((-_mi_numpy(t), oracle.pack_index(*q)) for t, q in zip(tabs, quads))
    idx, key = oracle.search_mi(d.geno, d.phen, top_k=8)
    np.testing.assert_allclose(key, [k[0] for k in keys[:8]], rtol=1e-9)
    # the same quads, up to near-ties the two rounding orders may swap
    assert set(int(v) for v in idx[:5]) <= set(k[1] for k in keys[:8])


# ---- chi-square objective ("e.g. mutual information, chi^2") ---------------------
def _chi2_scipy(t):
    """Pearson X^2 from scipy's textbook routine on the 2 x (non-empty cells) table, no continuity correction."""
    from scipy.stats import chi2_contingency
    t = np.asarray(t, dtype=np.float64)
    t = t[:, t.sum(axis=0) > 0]
    return float(chi2_contingency(t, correction=False)[0])


def test_chi2_matches_scipy_and_closed_forms():
    d = datagen.make_config("C1")
    quads = [[0, 1, 2, 3], [3, 11, 22, 35], [5, 9, 17, 30], [1, 20, 30, 39]]
    for t in oracle.tables(d.geno, d.phen, quads):
        want = _chi2_scipy(t)
        assert abs(oracle.chi2(t) - want) < 1e-10 * max(1.0, want)
    # unbalanced ragged workload (C5 shape, 30/70) on a few quads
    d5 = datagen.make_config("C5", n_snps=12)
    for t in oracle.tables(d5.geno, d5.phen, [[0, 1, 2, 3], [2, 5, 7, 11]]):
        want = _chi2_scipy(t)
        assert abs(oracle.chi2(t) - want) < 1e-10 * max(1.0, want)
    # independence: every non-empty cell split in the class ratio -> 0; perfect association -> M;
    # an empty phenotype -> 0 (defined, no variation)
    ind = np.zeros((2, 81), dtype=np.uint32)
    ind[0, :10], ind[1, :10] = 3, 1
    assert abs(oracle.chi2(ind)) < 1e-9
    perf = np.zeros((2, 81), dtype=np.uint32)
    perf[0, 0], perf[1, 80] = 30, 10
    assert abs(oracle.chi2(perf) - 40.0) < 1e-12
    one = np.zeros((2, 81), dtype=np.uint32)
    one[0, :5] = 7
    assert oracle.chi2(one) == 0.0
    # 2 x 2 textbook value: [[10, 20], [30, 40]] -> X^2 = 100 * (10*40 - 20*30)^2 / (30 * 70 * 40 * 60)
    tb = np.zeros((2, 81), dtype=np.uint32)
    tb[0, 4], tb[0, 60], tb[1, 4], tb[1, 60] = 10, 20, 30, 40
    assert abs(oracle.chi2(tb) - 100 * 200.0 ** 2 / (30 * 70 * 40 * 60)) < 1e-12


def test_chi2_search_equals_scipy_ranking():
    d = datagen.make_dataset(9, 20, 24, 5, planted=None, name="tinychi")
    quads = list(itertools.combinations(range(9), 4))
    tabs = oracle.tables(d.geno, d.phen, quads)
    keys = sorted((-_chi2_scipy(t), oracle.pack_index(*q)) for t, q in zip(tabs, quads))
    idx, key = oracle.search_chi2(d.geno, d.phen, top_k=8)
    np.testing.assert_allclose(key, [k[0] for k in keys[:8]], rtol=1e-9)
    assert set(int(v) for v in idx[:5]) <= set(k[1] for k in keys[:8])


def test_chi2_search_recovers_planted_quad():
    d = datagen.make_config("C1")
    idx, _ = oracle.search_chi2(d.geno, d.phen, top_k=1)
    assert oracle.unpack_index(int(idx[0])) == tuple(d.planted)


# ---- third-order search with the alternative objectives (NEXT-3 x NEXT-4) ---------------------------------
def test_triple_objectives_match_scipy_and_definition():
    d = datagen.make_config("C5", n_snps=10)
    for t in oracle.tables3(d.geno, d.phen, [[0, 1, 2], [2, 5, 9], [1, 4, 7]]):
        want = _chi2_scipy(t)
        assert abs(oracle.score3(t, "chi2") - want) < 1e-10 * max(1.0, want)
        want = _mi_numpy(t)
        assert abs(oracle.score3(t, "mi") - want) < 1e-9 * max(1.0, abs(want))


def test_triple_objective_search_equals_scipy_ranking():
    d = datagen.make_dataset(12, 30, 34, 8, planted=None, name="tiny3obj")
    tri = list(itertools.combinations(range(12), 3))
    tabs = oracle.tables3(d.geno, d.phen, tri)
    for obj, f in (("chi2", _chi2_scipy), ("mi", _mi_numpy)):
        keys = sorted((-f(t), oracle.pack_index(i, j, k, 0)) for t, (i, j, k) in zip(tabs, tri))
        idx, key = oracle.search3_obj(d.geno, d.phen, obj, top_k=8)
        np.testing.assert_allclose(key, [k[0] for k in keys[:8]], rtol=1e-9)
        assert set(int(v) for v in idx[:5]) <= set(k[1] for k in keys[:8])
