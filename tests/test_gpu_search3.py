"""Third-order search on the GPU (epi4_search3: the tensor-core 3-way-table mode with a scoring epilogue)
against the CPU oracle: top-k keys bit-identical (K2 summed in the same canonical order from the same
host-built lgamma table)."""
import numpy as np
import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("cfg,nsnp,k", [("C1", None, 64), ("C2", 64, 32), ("C5", 48, 32), ("C3", 150, 16)])
def test_search3_matches_oracle(cfg, nsnp, k):
    import paper_conf_icpp_nobreiss22_b200 as epi
    d = datagen.make_config(cfg, n_snps=nsnp)
    want_idx, want_k2 = oracle.search3(d.geno, d.phen, top_k=k)
    with epi.Epi4(0, pipe="tc") as e:
        e.load_genotypes(d.geno, d.phen)
        idx, k2 = e.search3(k)
        assert e.stats()["quads"] == d.n_snps * (d.n_snps - 1) * (d.n_snps - 2) // 6
    np.testing.assert_array_equal(idx, want_idx)
    np.testing.assert_array_equal(k2, want_k2)


def test_search3_rank_partition_merges():
    import paper_conf_icpp_nobreiss22_b200 as epi
    d = datagen.make_config("C2", n_snps=96)
    with epi.Epi4(0, pipe="tc") as e:
        e.load_genotypes(d.geno, d.phen)
        want = e.search3(16)
    parts = []
    for r in range(3):
        with epi.Epi4(0, pipe="tc", rank=r, world=3) as e:
            e.load_genotypes(d.geno, d.phen)
            parts.append(e.search3(16))
    idx, k2 = epi.merge_topk(parts, 16)
    np.testing.assert_array_equal(idx, want[0])
    np.testing.assert_array_equal(k2, want[1])
