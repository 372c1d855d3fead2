"""Pins for the CPU oracle (oracle/epi4_oracle.c) against things other than itself.

Each pin is chosen so that a plausible mistake in the oracle (dropped term, wrong sign,
wrong lgamma argument, transposed cell index, swapped phenotype rows, broken top-k order)
fails at least one of them:

* hand-enumerated dataset (tests/golden/hand_example.txt): exact cells and
  K2 = log 576 (closed form);
* closed forms: single-cell tables, all-samples-in-one-cell K2 = lgamma(M+2)-lgamma(n0+1)-lgamma(n1+1);
* invariants: cell sums equal n0 / n1 (unbalanced classes, so swapped rows fail);
  4-way -> 3-way / 2-way / 1-way marginalisation against a separately written numpy brute force;
  mathematical symmetries of K2 (case/control swap, SNP permutation, genotype relabelling);
* planted 4-way interaction recovered as the argmin (several seeds);
* top-k: brute-force enumeration + sort on tiny inputs; exact ties from duplicated SNPs resolve to
  the lexicographically smallest quad (reading #3).
"""
import itertools
import math
import os

import numpy as np
import pytest

import datagen
import oracle

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "hand_example.txt")


def _read_golden():
    samples, cells, planes = [], {}, {}
    with open(GOLDEN) as f:
        for line in f:
            line = line.split("#")[0].strip()
            if not line:
                continue
            tok = line.split()
            if tok[0] in ("control", "case"):
                samples.append((1 if tok[0] == "case" else 0, [int(v) for v in tok[1:]]))
            elif tok[0] == "cell":
                cells[int(tok[1])] = (int(tok[2]), int(tok[3]))
            elif tok[0] == "planes":
                planes[int(tok[1])] = tuple(int(v, 16) for v in tok[2:])
    geno = np.array([s[1] for s in samples], dtype=np.uint8).T.copy()
    phen = np.array([s[0] for s in samples], dtype=np.uint8)
    return geno, phen, cells, planes


# ---------------------------------------------------------------------------------------------
# independent numpy brute force for lower-order tables (not the oracle's code path)

def np_table(geno, phen, snps):
    """Brute-force len(snps)-way table via np.bincount -> [2, 3**len(snps)]."""
    code = np.zeros(geno.shape[1], dtype=np.int64)
    for s in snps:
        code = code * 3 + geno[s].astype(np.int64)
    size = 3 ** len(snps)
    return np.stack([np.bincount(code[phen == p], minlength=size) for p in (0, 1)])


# ---------------------------------------------------------------------------------------------

def test_hand_example_cells_and_k2():
    geno, phen, cells, _ = _read_golden()
    t = oracle.tables(geno, phen, [(0, 1, 2, 3)])[0]
    expect = np.zeros((2, 81), dtype=np.uint32)
    for c, (r0, r1) in cells.items():
        expect[0, c], expect[1, c] = r0, r1
    np.testing.assert_array_equal(t, expect)
    k2 = oracle.score(geno, phen, [(0, 1, 2, 3)])[0]
    assert abs(k2 - math.log(576.0)) <= 4 * np.spacing(math.log(576.0))
    # and the search over the only quad returns it
    idx, kv = oracle.search(geno, phen, top_k=3)
    assert len(idx) == 1 and oracle.unpack_index(idx[0]) == (0, 1, 2, 3) and kv[0] == k2


def test_hand_example_matches_datagen_copy():
    geno, phen, _, _ = _read_golden()
    d = datagen.hand_dataset()
    np.testing.assert_array_equal(d.geno, geno)
    np.testing.assert_array_equal(d.phen, phen)


@pytest.mark.parametrize("r0,r1,expect", [
    (0, 0, 0.0),                 # empty cell: log 1
    (1, 0, math.log(2)),         # log(2!/1!)
    (0, 1, math.log(2)),
    (1, 1, math.log(6)),         # log(3!/(1!1!))
    (2, 0, math.log(3)),         # log(3!/2!)
    (2, 1, math.log(12)),        # log(4!/(2!1!))
    (3, 3, math.log(5040 / 36)), # log(7!/(3!3!))
])
def test_k2_single_cell_closed_forms(r0, r1, expect):
    t = np.zeros((2, 81), dtype=np.uint32)
    t[0, 17], t[1, 17] = r0, r1
    assert abs(oracle.k2(t) - expect) <= 1e-13 * max(1.0, expect)


def test_k2_all_samples_one_cell_closed_form():
    # every genotype AA -> all samples fall into cell 0
    n0, n1 = 256, 256
    geno = np.zeros((5, n0 + n1), dtype=np.uint8)
    phen = np.array([0] * n0 + [1] * n1, dtype=np.uint8)
    k2 = oracle.score(geno, phen, [(0, 1, 2, 4)])[0]
    closed = math.lgamma(n0 + n1 + 2) - math.lgamma(n0 + 1) - math.lgamma(n1 + 1)
    assert abs(k2 - closed) <= 1e-12 * closed
    assert abs(k2 - 357.786190345759) < 1e-9   # SURVEY.md §8(c) printed value
    # a single aa-only cell (cell 80) gives the same value
    geno[:] = 2
    assert abs(oracle.score(geno, phen, [(0, 1, 2, 3)])[0] - closed) <= 1e-12 * closed


def _unbalanced(seed=7, n=9, n0=37, n1=23):
    return datagen.make_dataset(n, n0, n1, seed)


def test_cell_sums_equal_class_sizes():
    d = _unbalanced()
    quads = list(itertools.combinations(range(d.n_snps), 4))
    t = oracle.tables(d.geno, d.phen, quads)
    assert (t[:, 0, :].sum(axis=1) == d.n_controls).all()
    assert (t[:, 1, :].sum(axis=1) == d.n_cases).all()


def test_marginalisation_all_quads_C1():
    d = datagen.make_config("C1")
    n = d.n_snps
    quads = np.array(list(itertools.combinations(range(n), 4)), dtype=np.int32)
    t4 = oracle.tables(d.geno, d.phen, quads).reshape(-1, 2, 3, 3, 3, 3).astype(np.int64)
    assert t4.shape[0] == 91390
    t3 = {tr: np_table(d.geno, d.phen, tr).reshape(2, 3, 3, 3) for tr in itertools.combinations(range(n), 3)}
    t2 = {pr: np_table(d.geno, d.phen, pr).reshape(2, 3, 3) for pr in itertools.combinations(range(n), 2)}
    t1 = {s: np_table(d.geno, d.phen, (s,)) for s in range(n)}
    for qi, q in enumerate(quads):
        q = tuple(int(v) for v in q)
        tab = t4[qi]
        for ax in range(4):            # drop SNP q[ax] -> 3-way table of the other three
            rest = tuple(v for a, v in enumerate(q) if a != ax)
            np.testing.assert_array_equal(tab.sum(axis=1 + ax), t3[rest])
        np.testing.assert_array_equal(tab.sum(axis=(3, 4)), t2[(q[0], q[1])])
        np.testing.assert_array_equal(tab.sum(axis=(1, 2)), t2[(q[2], q[3])])
        np.testing.assert_array_equal(tab.sum(axis=(2, 4)), t2[(q[0], q[2])])
        np.testing.assert_array_equal(tab.sum(axis=(1, 2, 3)), t1[q[3]])


def test_full_table_vs_numpy_bruteforce_sampled():
    d = _unbalanced(seed=11, n=12, n0=101, n1=57)
    rng = np.random.default_rng(3)
    quads = [tuple(sorted(rng.choice(d.n_snps, 4, replace=False))) for _ in range(50)]
    t = oracle.tables(d.geno, d.phen, quads)
    for qi, q in enumerate(quads):
        np.testing.assert_array_equal(t[qi], np_table(d.geno, d.phen, q))


def test_k2_symmetries():
    d = _unbalanced(seed=5, n=8, n0=300, n1=200)
    quads = list(itertools.combinations(range(d.n_snps), 4))
    base = oracle.score(d.geno, d.phen, quads)
    # swap phenotype labels
    sw = oracle.score(d.geno, (1 - d.phen).astype(np.uint8), quads)
    np.testing.assert_allclose(sw, base, rtol=1e-12)
    # permute SNPs inside each quad (cells permute -> same multiset of terms)
    perm = oracle.score(d.geno, d.phen, [(q[3], q[1], q[0], q[2]) for q in quads])
    np.testing.assert_allclose(perm, base, rtol=1e-12)
    # relabel genotypes of SNP 0: 0 <-> 2
    g2 = d.geno.copy()
    g2[0] = (2 - g2[0]).astype(np.uint8)
    rel = oracle.score(g2, d.phen, quads)
    np.testing.assert_allclose(rel, base, rtol=1e-12)
    assert (base >= 0).all()


@pytest.mark.parametrize("seed", [1000, 1001, 1002, 1003])
def test_planted_recovery_C1(seed):
    d = datagen.make_config("C1", seed=seed)
    idx, k2v = oracle.search(d.geno, d.phen, top_k=2)
    assert oracle.unpack_index(idx[0]) == (3, 11, 22, 35)
    assert k2v[1] - k2v[0] > 20.0          # clear gap to the runner-up


def _numpy_k2(tab):
    # written independently of the C code (used only to pin the search's enumeration + ordering)
    s = 0.0
    for c in range(81):
        r0, r1 = int(tab[0, c]), int(tab[1, c])
        s += (math.lgamma(r0 + r1 + 2) - math.lgamma(r0 + 1)) - math.lgamma(r1 + 1)
    return s


def test_topk_matches_bruteforce_enumeration():
    d = _unbalanced(seed=21, n=9, n0=40, n1=35)
    quads = list(itertools.combinations(range(d.n_snps), 4))
    keys = sorted((_numpy_k2(np_table(d.geno, d.phen, q)), oracle.pack_index(*q)) for q in quads)
    for k in (1, 5, len(quads), len(quads) + 7):
        idx, k2v = oracle.search(d.geno, d.phen, top_k=k)
        assert len(idx) == min(k, len(quads))
        assert [int(v) for v in idx] == [kk[1] for kk in keys[:len(idx)]]
        np.testing.assert_allclose(k2v, [kk[0] for kk in keys[:len(idx)]], rtol=1e-12)
        assert (np.diff(k2v) >= 0).all()


def test_exact_ties_break_lexicographically():
    d = _unbalanced(seed=9, n=8, n0=64, n1=64)
    g = d.geno.copy()
    g[6] = g[2]              # SNP 6 duplicates SNP 2 -> quads swapping 2<->6 have identical tables
    g[7] = g[2]
    quads = list(itertools.combinations(range(8), 4))
    k2all = oracle.score(g, d.phen, quads)
    idx, k2v = oracle.search(g, d.phen, top_k=len(quads))
    # every run of equal K2 values is ordered by packed index
    for a in range(len(idx) - 1):
        if k2v[a] == k2v[a + 1]:
            assert idx[a] < idx[a + 1]
    # ties actually occur
    assert len(np.unique(k2all)) < len(quads)


def test_thread_count_independent():
    d = datagen.make_config("C1")
    a = oracle.search(d.geno, d.phen, top_k=25, n_threads=1)
    b = oracle.search(d.geno, d.phen, top_k=25, n_threads=4)
    np.testing.assert_array_equal(a[0], b[0])
    np.testing.assert_array_equal(a[1], b[1])


def test_rejects_bad_genotypes():
    geno = np.zeros((4, 8), dtype=np.uint8)
    geno[1, 3] = 3
    with pytest.raises(ValueError):
        oracle.score(geno, np.zeros(8, dtype=np.uint8), [(0, 1, 2, 3)])
