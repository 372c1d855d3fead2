"""GPU parity: libepi4 (through the C ABI) against the CPU oracle on the same seeded inputs.

Bars (BASELINE.json north_star): contingency counts bit-exact; argmin / top-k quads bit-exact with
lexicographic tie-break; K2 within 1e-9 relative (asserted here: bit-identical, because both sides
add the same doubles in the same order, reading #4).
"""
import functools
import itertools

import numpy as np
import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu

PIPES = ["lop3", "tc", "tc224"]   # tc: the tile geometry the load picks (N = 128 for these sample counts)
PIPES_GEOM = ["lop3", "tc128", "tc224"]   # both tensor-core geometries forced


def _epi():
    import paper_conf_icpp_nobreiss22_b200 as epi
    return epi


def _engine(pipe="tc", **kw):
    """pipe: lop3, tc (geometry chosen by the load), tc128 / tc224 (geometry forced, opts.flags)"""
    if pipe in ("tc128", "tc224"):
        kw["tile"] = int(pipe[2:])
        pipe = "tc"
    return _epi().Epi4(0, pipe=pipe, **kw)


def np_pack(geno, phen):
    """Trivial reference packer: per phenotype, samples in order, LSB-first, rows 2*snp+g."""
    out = []
    for p in (0, 1):
        g = geno[:, phen == p]
        n, m = g.shape
        wp = (m + 31) // 32
        rows = np.zeros((2 * n, wp), dtype=np.uint32)
        for gv in (0, 1):
            bits = (g == gv).astype(np.uint64)
            padded = np.zeros((n, wp * 32), dtype=np.uint64)
            padded[:, :m] = bits
            words = (padded.reshape(n, wp, 32) << np.arange(32, dtype=np.uint64)).sum(axis=2)
            rows[gv::2] = words.astype(np.uint32)
        out.append(rows)
    return out


def all_quads(n):
    return np.array(list(itertools.combinations(range(n), 4)), dtype=np.int64)


def packq(q):
    q = np.asarray(q, dtype=np.uint64)
    return (q[:, 0] << np.uint64(48)) | (q[:, 1] << np.uint64(32)) | (q[:, 2] << np.uint64(16)) | q[:, 3]


# ---- pack / load ----------------------------------------------------------------------------------

@pytest.mark.parametrize("n,n0,n1", [(40, 256, 256), (7, 333, 667), (5, 1, 1), (9, 128, 129), (64, 4097, 31)])
def test_pack_matches_reference_packer(n, n0, n1):
    d = datagen.make_dataset(n, n0, n1, seed=n + n0)
    with _engine() as e:
        e.load_genotypes(d.geno, d.phen)
        ref = np_pack(d.geno, d.phen)
        got = [np.zeros_like(ref[0]), np.zeros_like(ref[1])]
        _epi().binding.epi4_get_bits(e.ctx, got[0], got[1])
        np.testing.assert_array_equal(got[0], ref[0])
        np.testing.assert_array_equal(got[1], ref[1])
        for r in got:
            assert not (r[0::2] & r[1::2]).any()       # AA & Aa == 0


def test_load_bits_equals_pack_and_validates():
    epi = _epi()
    d = datagen.make_dataset(12, 300, 200, seed=4)
    ref = np_pack(d.geno, d.phen)
    with _engine() as e:
        e.load_bits(ref[0], ref[1], 12, 300, 200)
        got = [np.zeros_like(ref[0]), np.zeros_like(ref[1])]
        epi.binding.epi4_get_bits(e.ctx, got[0], got[1])
        np.testing.assert_array_equal(got[0], ref[0])
        bad = ref[0].copy()
        bad[3, -1] |= np.uint32(1 << 31)                  # pad bit beyond n0 = 300
        with pytest.raises(epi.Epi4Error) as ei:
            e.load_bits(bad, ref[1], 12, 300, 200)
        assert ei.value.code == epi.binding.EPI4_EINVAL
        bad = ref[1].copy()
        bad[0, 0] |= bad[1, 0] | np.uint32(1)             # AA & Aa overlap
        bad[1, 0] |= np.uint32(1)
        with pytest.raises(epi.Epi4Error):
            e.load_bits(ref[0], bad, 12, 300, 200)
        g = d.geno.copy()
        g[5, 17] = 3
        with pytest.raises(epi.Epi4Error):
            e.load_genotypes(g, d.phen)


def test_errors_state_and_range():
    epi = _epi()
    with _engine() as e:
        with pytest.raises(epi.Epi4Error) as ei:
            e.search(1)
        assert ei.value.code == epi.binding.EPI4_ESTATE
        d = datagen.make_config("C1")
        e.load_genotypes(d.geno, d.phen)
        for k in (0, 1025):
            with pytest.raises(epi.Epi4Error):
                e.search(k)


# ---- tables -----------------------------------------------------------------------------------------

def test_tables_all_quads_C1():
    d = datagen.make_config("C1")
    q = all_quads(d.n_snps)
    ref = oracle.tables(d.geno, d.phen, q)
    with _engine() as e:
        e.load_genotypes(d.geno, d.phen)
        got = e.tables(packq(q))
        np.testing.assert_array_equal(got, ref)
        # any SNP order is accepted and used as given
        rng = np.random.default_rng(0)
        qp = np.array([rng.permutation(row) for row in q[:2000]])
        np.testing.assert_array_equal(e.tables(packq(qp)), oracle.tables(d.geno, d.phen, qp))


# ---- search on C1 -------------------------------------------------------------------------------------

@pytest.mark.parametrize("pipe", PIPES)
def test_search_C1_topk_bit_exact(pipe):
    d = datagen.make_config("C1")
    ref_idx, ref_k2 = oracle.search(d.geno, d.phen, top_k=64)
    with _engine(pipe) as e:
        e.load_genotypes(d.geno, d.phen)
        idx, k2 = e.search(64)
        assert e.stats()["quads"] == 91390
    np.testing.assert_array_equal(idx, ref_idx)
    np.testing.assert_array_equal(k2, ref_k2)           # bit-identical doubles
    assert _epi().unpack_index(idx[0]) == (3, 11, 22, 35)


@pytest.mark.parametrize("pipe", PIPES)
def test_search_dump_all_counts_C1(pipe):
    import torch
    d = datagen.make_config("C1")
    n = d.n_snps
    q = all_quads(n)
    ref = oracle.tables(d.geno, d.phen, q)      # lexicographic order == colex rank order? no: map below
    rank = (q[:, 3] * (q[:, 3] - 1) * (q[:, 3] - 2) * (q[:, 3] - 3) // 24 + q[:, 2] * (q[:, 2] - 1) * (q[:, 2] - 2) // 6
            + q[:, 1] * (q[:, 1] - 1) // 2 + q[:, 0])
    buf = torch.full((len(q), 162), 0xFFFFFFFF, dtype=torch.int64).to(torch.int32).cuda()
    with _engine(pipe) as e:
        e.load_genotypes(d.geno, d.phen)
        _epi().binding.epi4_set_dump(e.ctx, buf)
        e.search(4)
        _epi().binding.epi4_set_dump(e.ctx, None)
    got = buf.cpu().numpy().view(np.uint32).reshape(-1, 2, 81)
    np.testing.assert_array_equal(got[rank], ref)


@pytest.mark.parametrize("pipe", PIPES)
def test_exact_ties_resolve_lexicographically(pipe):
    d = datagen.make_config("C1", seed=77)
    g = d.geno.copy()
    g[20] = g[3]
    g[30] = g[3]
    g[36] = g[11]
    ref_idx, ref_k2 = oracle.search(g, d.phen, top_k=200)
    assert len(np.unique(ref_k2)) < len(ref_k2)
    with _engine(pipe) as e:
        e.load_genotypes(g, d.phen)
        idx, k2 = e.search(200)
    np.testing.assert_array_equal(idx, ref_idx)
    np.testing.assert_array_equal(k2, ref_k2)


@pytest.mark.parametrize("pipe", PIPES)
@pytest.mark.parametrize("n,n0,n1", [(4, 4, 4), (5, 3, 2), (6, 1, 1), (35, 128, 128), (33, 129, 255), (37, 700, 300)])
def test_small_and_ragged_shapes(pipe, n, n0, n1):
    d = datagen.make_dataset(n, n0, n1, seed=3 * n + n0)
    k = 30
    ref_idx, ref_k2 = oracle.search(d.geno, d.phen, top_k=k)
    with _engine(pipe) as e:
        e.load_genotypes(d.geno, d.phen)
        idx, k2 = e.search(k)
    np.testing.assert_array_equal(idx, ref_idx)
    np.testing.assert_array_equal(k2, ref_k2)


def test_hand_example_on_gpu():
    d = datagen.hand_dataset()
    with _engine() as e:
        e.load_genotypes(d.geno, d.phen)
        idx, k2 = e.search(5)
        t = e.tables(packq([[0, 1, 2, 3]]))
    assert len(idx) == 1 and _epi().unpack_index(idx[0]) == (0, 1, 2, 3)
    assert abs(k2[0] - np.log(576.0)) < 1e-13
    np.testing.assert_array_equal(t, oracle.tables(d.geno, d.phen, [(0, 1, 2, 3)]))


# ---- configs C2..C5: sub-windows at full M and sampled quads at full N ---------------------------------

WINDOWS = {"C2": 64, "C3": 64, "C4": 64, "C5": 64}


@functools.lru_cache(maxsize=None)
def _subwindow_ref(cfg):
    d = datagen.make_config(cfg, n_snps=WINDOWS[cfg], planted=False)
    idx, k2 = oracle.search(d.geno, d.phen, top_k=32)
    return d, idx, k2


@pytest.mark.parametrize("pipe", PIPES_GEOM)
@pytest.mark.parametrize("cfg", ["C2", "C3", "C4", "C5"])
def test_subwindow_full_samples(cfg, pipe):
    """First W SNPs of the config's dataset with all M samples (ragged 100003 in C5)."""
    w = WINDOWS[cfg]
    d, ref_idx, ref_k2 = _subwindow_ref(cfg)
    with _engine(pipe) as e:
        e.load_genotypes(d.geno, d.phen)
        idx, k2 = e.search(32)
        rng = np.random.default_rng(1)
        q = np.sort(np.array([rng.choice(w, 4, replace=False) for _ in range(300)]), axis=1)
        np.testing.assert_array_equal(e.tables(packq(q)), oracle.tables(d.geno, d.phen, q))
    np.testing.assert_array_equal(idx, ref_idx)
    np.testing.assert_array_equal(k2, ref_k2)


def _sample_quads(n, rng, count):
    qs = [np.sort(rng.choice(n, 4, replace=False)) for _ in range(count)]
    # diagonal-block and block-edge quads, last SNPs
    for b in range(0, n - 64, max(32, (n // 8) // 32 * 32)):
        qs.append(np.array([b, b + 1, b + 2, b + 3]))
        qs.append(np.array([b + 30, b + 31, b + 32, b + 33]))
        qs.append(np.array([b, b + 31, b + 32, b + 63]))
    qs.append(np.array([n - 4, n - 3, n - 2, n - 1]))
    qs.append(np.array([0, 1, n - 2, n - 1]))
    return np.array(qs, dtype=np.int64)


@pytest.mark.parametrize("cfg", ["C2", "C5", "C3"])
def test_full_size_sampled_tables(cfg):
    d = datagen.make_config(cfg)
    rng = np.random.default_rng(5)
    q = _sample_quads(d.n_snps, rng, 400)
    with _engine() as e:
        e.load_genotypes(d.geno, d.phen)
        got = e.tables(packq(q))
    np.testing.assert_array_equal(got, oracle.tables(d.geno, d.phen, q))


@pytest.mark.parametrize("pipe", PIPES)
def test_full_C2_units_sample_and_planted(pipe):
    """C2 at full size in the bench's launch configuration: a bounded slice of the plan's units is
    checked quad-by-quad against the oracle, and the full search's argmin is the planted quad with
    K2 values the oracle reproduces bit-exactly."""
    epi = _epi()
    d = datagen.make_config("C2")
    n = d.n_snps
    units, _ = epi.binding.epi4_plan_units(n, 0, 1)
    # a few units from the end of the plan (small ones), enumerated explicitly
    sel = range(len(units) - 6, len(units))
    quads = []
    for u in sel:
        wb, x = (int(v) for v in units[u])
        for w in range(128 * wb, min(128 * wb + 128, x)):
            for y in range(x + 1, n):
                for z in range(y + 1, n):
                    quads.append((w, x, y, z))
    quads = np.array(quads, dtype=np.int32)
    ref_k2 = oracle.score(d.geno, d.phen, quads)
    ref_idx = packq(quads)
    order = np.lexsort((ref_idx, ref_k2))[:16]
    with _engine(pipe) as e:
        e.load_genotypes(d.geno, d.phen)
        idx, k2 = e.search_units(len(units) - 6, len(units), 16)
        np.testing.assert_array_equal(idx, ref_idx[order])
        np.testing.assert_array_equal(k2, ref_k2[order])
        idx, k2 = e.search(8)
    assert epi.unpack_index(idx[0]) == datagen.planted_quad_for(n)
    qs = np.array([epi.unpack_index(v) for v in idx], dtype=np.int32)
    np.testing.assert_array_equal(k2, oracle.score(d.geno, d.phen, qs))


@pytest.mark.parametrize("cfg", ["C5", "C2"])
def test_fp32_filter_keeps_exact_topk(cfg):
    """The tensor-core epilogue scores a quad exactly only when its fp32 Stirling lower bound can beat the
    CTA's k-th best K2 (epilogue.cuh, reading #16).  With a large k (a loose threshold for most
    of the run) and the largest M (C5, the widest rounding bound), the top-1024 must equal both the
    oracle's and the unfiltered run's (debug flag 16: exact K2 for every quad)."""
    w = WINDOWS[cfg]
    d = datagen.make_config(cfg, n_snps=w, planted=False)
    ref_idx, ref_k2 = oracle.search(d.geno, d.phen, top_k=1024)
    with _engine("tc") as e:
        e.load_genotypes(d.geno, d.phen)
        idx, k2 = e.search(1024)
        n_exact = e.stats()["prof"][0]
    with _engine("tc", debug=16) as e:
        e.load_genotypes(d.geno, d.phen)
        idx_u, k2_u = e.search(1024)
    np.testing.assert_array_equal(idx, ref_idx)
    np.testing.assert_array_equal(k2, ref_k2)
    np.testing.assert_array_equal(idx_u, ref_idx)
    np.testing.assert_array_equal(k2_u, ref_k2)
    assert 1024 <= n_exact < len(all_quads(w))          # the filter did filter
