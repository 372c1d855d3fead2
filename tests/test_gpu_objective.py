"""Alternative objective: the search ranked by mutual information (EPI4_OBJ_MI),
scored exactly for every quad on the GPU from the same host-built k ln k table and in the same canonical
order as the oracle, so the keys are bit-identical; both pipes.  The same for Pearson chi-square
(EPI4_OBJ_CHI2): exact integer numerators and one correctly rounded division per cell on both sides."""
import numpy as np
import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("pipe", ["tc", "lop3"])
@pytest.mark.parametrize("cfg,nsnp", [("C1", None), ("C5", 24)])
def test_mi_search_matches_oracle(pipe, cfg, nsnp):
    import paper_conf_icpp_nobreiss22_b200 as epi
    d = datagen.make_config(cfg, n_snps=nsnp)
    want_idx, want_key = oracle.search_mi(d.geno, d.phen, top_k=32)
    with epi.Epi4(0, pipe=pipe, objective="mi") as e:
        e.load_genotypes(d.geno, d.phen)
        idx, key = e.search(32)
    np.testing.assert_array_equal(idx, want_idx)
    np.testing.assert_array_equal(key, want_key)


@pytest.mark.parametrize("pipe", ["tc", "lop3"])
@pytest.mark.parametrize("cfg,nsnp", [("C1", None), ("C5", 24)])
def test_chi2_search_matches_oracle(pipe, cfg, nsnp):
    import paper_conf_icpp_nobreiss22_b200 as epi
    d = datagen.make_config(cfg, n_snps=nsnp)
    want_idx, want_key = oracle.search_chi2(d.geno, d.phen, top_k=32)
    with epi.Epi4(0, pipe=pipe, objective="chi2") as e:
        e.load_genotypes(d.geno, d.phen)
        idx, key = e.search(32)
    np.testing.assert_array_equal(idx, want_idx)
    np.testing.assert_array_equal(key, want_key)


def test_chi2_planted_quad_on_a_multi_tile_problem():
    """N = 160 (several 128-SNP w-ranges, a ragged tail): the chi-square search's best quad is the planted one
    and its key equals the oracle's chi-square of the oracle's table for that quad."""
    import paper_conf_icpp_nobreiss22_b200 as epi
    d = datagen.make_dataset(160, 4096, 4096, 77, planted=datagen.planted_quad_for(160), name="chi2-160")
    with epi.Epi4(0, pipe="tc", objective="chi2") as e:
        e.load_genotypes(d.geno, d.phen)
        idx, key = e.search(4)
    best = oracle.unpack_index(int(idx[0]))
    assert best == tuple(d.planted)
    t = oracle.tables(d.geno, d.phen, [list(best)])[0]
    assert key[0] == -oracle.chi2(t)


@pytest.mark.parametrize("objective", ["chi2", "mi"])
@pytest.mark.parametrize("cfg,nsnp,k", [("C5", 32, 64), ("C2", 48, 1024)])
def test_fp32_objective_filter_keeps_exact_topk(objective, cfg, nsnp, k):
    """The tensor-core epilogue scores a quad's exact chi-square / MI only when its fp32 upper bound on X^2 /
    M*I can beat the CTA's k-th best key (epilogue.cuh, cell_chi_acc / cell_mi_acc).  With a large k (a loose threshold for most of the
    run) and the largest M (C5, unbalanced), the top-k must equal the oracle's and the unfiltered run's
    (debug flag 16: exact score for every quad), and the filter must have skipped quads."""
    import paper_conf_icpp_nobreiss22_b200 as epi
    d = datagen.make_config(cfg, n_snps=nsnp, planted=False)
    ref_idx, ref_key = (oracle.search_chi2 if objective == "chi2" else oracle.search_mi)(d.geno, d.phen, top_k=k)
    with epi.Epi4(0, pipe="tc", objective=objective) as e:
        e.load_genotypes(d.geno, d.phen)
        idx, key = e.search(k)
        n_exact = e.stats()["prof"][0]
    with epi.Epi4(0, pipe="tc", objective=objective, debug=16) as e:
        e.load_genotypes(d.geno, d.phen)
        idx_u, key_u = e.search(k)
    np.testing.assert_array_equal(idx, ref_idx)
    np.testing.assert_array_equal(key, ref_key)
    np.testing.assert_array_equal(idx_u, ref_idx)
    np.testing.assert_array_equal(key_u, ref_key)
    nq = nsnp * (nsnp - 1) * (nsnp - 2) * (nsnp - 3) // 24
    assert k <= n_exact < nq


@pytest.mark.parametrize("objective", ["mi", "chi2"])
@pytest.mark.parametrize("cfg,nsnp,k", [("C1", None, 64), ("C5", 40, 32), ("C2", 100, 16)])
def test_search3_objectives_match_oracle(objective, cfg, nsnp, k):
    """Third-order search ranked by MI / chi-square: keys bit-identical to oracle.search3_obj."""
    import paper_conf_icpp_nobreiss22_b200 as epi
    d = datagen.make_config(cfg, n_snps=nsnp)
    want_idx, want_key = oracle.search3_obj(d.geno, d.phen, objective, top_k=k)
    with epi.Epi4(0, pipe="tc", objective=objective) as e:
        e.load_genotypes(d.geno, d.phen)
        idx, key = e.search3(k)
    np.testing.assert_array_equal(idx, want_idx)
    np.testing.assert_array_equal(key, want_key)


def test_chi2_rejects_counts_whose_numerator_is_not_exact():
    """EPI4_OBJ_CHI2 needs n0 n1 M < 2^53 (exact uint64 -> double numerators, include/epi4.h): at n0 = 4e6,
    n1 = 1000 (packable: 22 + 10 bits) the product is 1.6e16, so the load fails for chi-square, not for K2."""
    import paper_conf_icpp_nobreiss22_b200 as epi
    n0, n1 = 4_000_000, 1000
    rng = np.random.default_rng(5)
    geno = rng.integers(0, 3, size=(4, n0 + n1), dtype=np.uint8)
    phen = np.zeros(n0 + n1, dtype=np.uint8)
    phen[:n1] = 1
    with epi.Epi4(0, pipe="tc", objective="chi2") as e:
        with pytest.raises(epi.Epi4Error):
            e.load_genotypes(geno, phen)
    with epi.Epi4(0, pipe="tc", objective="k2") as e:
        e.load_genotypes(geno, phen)
        idx, _ = e.search(1)
        assert len(idx) == 1
