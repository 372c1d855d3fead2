"""Alternative objective: the search ranked by mutual information (EPI4_OBJ_MI),
scored exactly for every quad on the GPU from the same host-built k ln k table and in the same canonical
order as the oracle, so the keys are bit-identical; both pipes."""
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


def test_mi_objective_rejected_by_the_third_order_search():
    import paper_conf_icpp_nobreiss22_b200 as epi
    d = datagen.make_config("C1")
    with epi.Epi4(0, pipe="tc", objective="mi") as e:
        e.load_genotypes(d.geno, d.phen)
        with pytest.raises(epi.Epi4Error):
            e.search3(4)
