"""Windowed 3-way table (tensor-core pipe): instead of all C(N,3) triples, two slabs FIRST(R) and
FIRST(X) of 128 x C(N,2) triples are rebuilt on the tensor cores while the search walks the units grouped by
(w-range, x-range).  Forced on small problems, it must reproduce the resident-table search exactly: every one
of the 162 counts of every quad (search dump) and the top-k keys."""
import numpy as np
import pytest

import datagen
import oracle

pytestmark = pytest.mark.gpu


def _epi():
    import paper_conf_icpp_nobreiss22_b200 as epi
    return epi


@pytest.mark.parametrize("cfg,nsnp,k", [("C1", None, 32), ("C2", 300, 64), ("C5", 200, 64)])
def test_windowed_t3_search_equals_resident(cfg, nsnp, k):
    epi = _epi()
    d = datagen.make_config(cfg, n_snps=nsnp)
    with epi.Epi4(0, pipe="tc") as e:
        e.load_genotypes(d.geno, d.phen)
        want = e.search(k)
    with epi.Epi4(0, pipe="tc", t3_windowed=True) as e:
        e.load_genotypes(d.geno, d.phen)
        with pytest.raises(epi.Epi4Error):          # the verification tables need the resident table
            e.tables(np.array([epi.pack_index(0, 1, 2, 3)], dtype=np.uint64))
        got = e.search(k)
    np.testing.assert_array_equal(got[0], want[0])
    np.testing.assert_array_equal(got[1], want[1])


def test_windowed_t3_dump_all_counts_C1_and_multi_range():
    """All 162 counts of every quad from the windowed search, against the oracle: C1 (one w-range) and a
    160-SNP problem (two w-ranges, so FIRST(X) != FIRST(R) slabs are exercised), sampled there."""
    import torch
    epi = _epi()
    for cfg, nsnp in (("C1", None), ("C2", 160)):
        d = datagen.make_config(cfg, n_snps=nsnp)
        n = d.n_snps
        tot = n * (n - 1) * (n - 2) * (n - 3) // 24
        buf = torch.zeros((tot, 162), dtype=torch.int32, device="cuda")
        with epi.Epi4(0, pipe="tc", t3_windowed=True) as e:
            e.load_genotypes(d.geno, d.phen)
            epi.binding.epi4_set_dump(e.ctx, buf)
            e.search(4)
            epi.binding.epi4_set_dump(e.ctx, None)
        got = buf.cpu().numpy().view(np.uint32).reshape(-1, 2, 81)
        rng = np.random.default_rng(11)
        q = np.array(sorted({tuple(sorted(rng.choice(n, 4, replace=False))) for _ in range(3000)}), dtype=np.int64)
        if cfg == "C1":
            import itertools
            q = np.array(list(itertools.combinations(range(n), 4)), dtype=np.int64)
        rank = (q[:, 3] * (q[:, 3] - 1) * (q[:, 3] - 2) * (q[:, 3] - 3) // 24
                + q[:, 2] * (q[:, 2] - 1) * (q[:, 2] - 2) // 6 + q[:, 1] * (q[:, 1] - 1) // 2 + q[:, 0])
        ref = oracle.tables(d.geno, d.phen, q.astype(np.int32))
        np.testing.assert_array_equal(got[rank], ref)
