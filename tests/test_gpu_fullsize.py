"""Parity of the PRODUCT path at full size (SURVEY.md §8(c) parity tiers 2-3).

The tensor-core search kernel itself records a hash-selected sample of the quads it evaluates (epi4_set_sample:
packed index, exact key, 2 x 81 counts from its own contraction + aa recovery + lower-order tables); every
recorded quad is compared with the oracle's per-sample brute force (oracle.tables) and its K2
with oracle.score (bit-identical doubles, reading #4).  Each search runs in the bench's launch
configuration (default grid, the full plan) on the BASELINE.json configs, so the sample spans diagonal blocks,
the last SNPs, the ragged last sample word, and (C3, C4) triple ranks beyond 2^32 entries of T3.
"""
import numpy as np
import pytest

import datagen
import oracle
from sampling import pack, rate_for, sampled, unpack

pytestmark = pytest.mark.gpu


def _epi():
    import paper_conf_icpp_nobreiss22_b200 as epi
    return epi


def comb4(n):
    return n * (n - 1) * (n - 2) * (n - 3) // 24


def _check_sample(d, q, keys, counts):
    quads = unpack(q)
    assert (np.diff(quads, axis=1) > 0).all() and quads[:, 3].max() < d.n_snps
    np.testing.assert_array_equal(counts, oracle.tables(d.geno, d.phen, quads))
    np.testing.assert_array_equal(keys, oracle.score(d.geno, d.phen, quads))
    return quads


def _coverage(quads, n):
    """The sample must reach the edges of the tiling, not just its bulk."""
    blk = 64
    return {
        "diag_wx": bool(((quads[:, 0] // blk) == (quads[:, 1] // blk)).any()),
        "adjacent_yz": bool((quads[:, 3] == quads[:, 2] + 1).any()),
        "high_z": bool((quads[:, 3] >= n - 16).any()),
        "low_w": bool((quads[:, 0] < 16).any()),
    }


def test_sample_is_exactly_the_predicted_set_C1():
    """Every quad of C1 whose hash hits is recorded once, and nothing else (the kernel evaluates every quad)."""
    from test_gpu_parity import all_quads
    d = datagen.make_config("C1")
    allq = all_quads(d.n_snps)
    want = np.sort(pack(allq)[sampled(pack(allq), 3, 12345)])
    for pipe in ("tc", "lop3"):
        with _epi().Epi4(0, pipe=pipe) as e:
            e.load_genotypes(d.geno, d.phen)
            e.set_sample(3, 12345, capacity=len(allq))
            e.search(16)
            q, k, c, n = e.get_sample()
        assert n == len(want)
        np.testing.assert_array_equal(np.sort(q), want)
        _check_sample(d, q, k, c)


@pytest.mark.parametrize("cfg", ["C2", "C5", "C3"])
def test_full_search_sampled_tables_and_planted(cfg):
    """Full search of the config (the bench's step minus the timing): >= 1e4 sampled quads bit-exact, the
    argmin is the planted quad, and the top-16 keys are the oracle's K2 of those quads (tier 2 + tier 3)."""
    epi = _epi()
    d = datagen.make_config(cfg)
    n = d.n_snps
    r = rate_for(comb4(n), 15000)
    with epi.Epi4(0, pipe="tc") as e:
        e.load_genotypes(d.geno, d.phen)
        e.set_sample(r, 2024 + n, capacity=1 << 16)
        idx, k2 = e.search(16)
        q, k, c, hits = e.get_sample()
        st = e.stats()
    assert st["quads"] == comb4(n)
    assert hits == len(q) >= 10000
    quads = _check_sample(d, q, k, c)
    assert all(_coverage(quads, n).values()), _coverage(quads, n)
    assert tuple(unpack(idx[:1])[0]) == datagen.planted_quad_for(n)
    np.testing.assert_array_equal(k2, oracle.score(d.geno, d.phen, unpack(idx)))
    assert (np.diff(k2) >= 0).all()
    assert k2[-1] <= k.min()              # nothing sampled beats the reported top-16


def _unit_index(units, wr, x):
    hit = np.nonzero((units[:, 0] == wr) & (units[:, 1] == x))[0]
    assert len(hit) == 1
    return int(hit[0])


def test_C4_windowed_slice_sampled_and_planted():
    """C4 (N=4096, M=65536) selects the windowed 3-way table: a slice of the plan around the
    planted quad's unit, spanning several w-ranges and a diagonal unit, checked on >= 1e4 sampled quads; the
    slice's argmin is the planted quad."""
    epi = _epi()
    d = datagen.make_config("C4")
    n = d.n_snps
    pq = datagen.planted_quad_for(n)
    units, cost = epi.binding.epi4_plan_units(n, 0, 1)
    wr_size = 64 if units[:, 0].max() >= (n + 127) // 128 else 128
    u0 = _unit_index(units, pq[0] // wr_size, pq[1])
    lo, hi = max(0, u0 - 12), min(len(units), u0 + 12)
    sel = units[lo:hi]
    assert len(set(sel[:, 0].tolist())) >= 3 and (sel[:, 1] // wr_size == sel[:, 0]).any()
    nq = sum(min(wr_size, int(x) - int(wr) * wr_size) * (n - int(x) - 1) * (n - int(x) - 2) // 2 for wr, x in sel)
    r = rate_for(nq, 15000)
    with epi.Epi4(0, pipe="tc") as e:
        e.load_genotypes(d.geno, d.phen)
        e.set_sample(r, 77, capacity=1 << 16)
        idx, k2 = e.search_units(lo, hi, 8)
        q, k, c, hits = e.get_sample()
        assert e.stats()["quads"] == nq
    assert hits == len(q) >= 10000
    _check_sample(d, q, k, c)
    assert tuple(unpack(idx[:1])[0]) == pq
    np.testing.assert_array_equal(k2, oracle.score(d.geno, d.phen, unpack(idx)))


def _worst_case(n=40, n0=70002, n1=30001, seed=9):
    """C5's class sizes with monomorphic SNPs: 0-3 all AA (quad 0,1,2,3 puts every sample in one cell: the
    largest fp32 accumulator values and the full packed-count field widths), 4-5 all Aa, 6 all aa."""
    d = datagen.make_dataset(n, n0, n1, seed=seed)
    g = d.geno.copy()
    g[0:4] = 0
    g[4:6] = 1
    g[6] = 2
    return datagen.Dataset(geno=g, phen=d.phen, n_controls=n0, n_cases=n1, planted=None, seed=seed, name="worst")


@pytest.mark.parametrize("pipe", ["tc", "tc128", "lop3"])   # tc: N = 224 is picked for 70002 controls
def test_worst_case_all_samples_in_one_cell(pipe):
    from test_gpu_parity import all_quads
    d = _worst_case()
    allq = all_quads(d.n_snps)
    ref_idx, ref_k2 = oracle.search(d.geno, d.phen, top_k=256)
    from test_gpu_parity import _engine
    with _engine(pipe) as e:
        e.load_genotypes(d.geno, d.phen)
        e.set_sample(0, 0, capacity=len(allq))          # every quad
        idx, k2 = e.search(256)
        q, k, c, n = e.get_sample()
    assert n == len(allq)
    np.testing.assert_array_equal(idx, ref_idx)
    np.testing.assert_array_equal(k2, ref_k2)
    order = np.argsort(q)
    q, k, c = q[order], k[order], c[order]
    np.testing.assert_array_equal(q, np.sort(pack(allq)))
    _check_sample(d, q, k, c)
    row = int(np.searchsorted(q, pack([[0, 1, 2, 3]])[0]))
    assert c[row, 0, 0] == 70002 and c[row, 1, 0] == 30001


def test_uniform_genotypes_full_C2():
    """Sensitivity run: uniform {0,1,2} genotypes at C2's shape; full search sampled, its
    top-16 re-scored by the oracle, and the first 64 SNPs searched against the oracle's exhaustive top-k."""
    epi = _epi()
    d = datagen.make_config("C2", uniform=True, planted=False)
    n = d.n_snps
    with epi.Epi4(0, pipe="tc") as e:
        e.load_genotypes(d.geno, d.phen)
        e.set_sample(rate_for(comb4(n), 12000), 5, capacity=1 << 15)
        idx, k2 = e.search(16)
        q, k, c, hits = e.get_sample()
    assert len(q) >= 10000
    _check_sample(d, q, k, c)
    np.testing.assert_array_equal(k2, oracle.score(d.geno, d.phen, unpack(idx)))
    w = datagen.make_config("C2", uniform=True, planted=False, n_snps=64)
    ref_idx, ref_k2 = oracle.search(w.geno, w.phen, top_k=32)
    with epi.Epi4(0, pipe="tc") as e:
        e.load_genotypes(w.geno, w.phen)
        idx, k2 = e.search(32)
    np.testing.assert_array_equal(idx, ref_idx)
    np.testing.assert_array_equal(k2, ref_k2)


@pytest.mark.parametrize("pipe", ["tc", "tc128", "lop3"])   # tc: N = 224 is picked for wide counts
@pytest.mark.parametrize("n0,n1", [(91750, 39322), (262144, 262144)])
def test_wide_counts_beyond_32_packed_bits(pipe, n0, n1):
    """bits(n0) + bits(n1) > 32 (the C5 sweep's M = 131072 at 30/70; the paper's 2048 x 524288 shape):
    64-bit packed counts through tables, contraction and epilogue.  Every quad's 2 x 81 table and the top-k
    against the oracle on a 24-SNP window."""
    from test_gpu_parity import all_quads
    d = datagen.make_dataset(24, n0, n1, seed=n0 + 7, planted=(2, 9, 15, 21))
    allq = all_quads(d.n_snps)
    ref_idx, ref_k2 = oracle.search(d.geno, d.phen, top_k=128)
    from test_gpu_parity import _engine
    with _engine(pipe) as e:
        e.load_genotypes(d.geno, d.phen)
        e.set_sample(0, 0, capacity=len(allq))
        idx, k2 = e.search(128)
        q, k, c, n = e.get_sample()
        t = e.tables(pack(allq[:500]))
    np.testing.assert_array_equal(idx, ref_idx)
    np.testing.assert_array_equal(k2, ref_k2)
    assert tuple(unpack(idx[:1])[0]) == (2, 9, 15, 21)
    assert n == len(allq)
    order = np.argsort(q)
    _check_sample(d, q[order], k[order], c[order])
    np.testing.assert_array_equal(t, oracle.tables(d.geno, d.phen, allq[:500]))
