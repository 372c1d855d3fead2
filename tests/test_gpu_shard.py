"""Sharded 3-way table (multi-GPU path) on one GPU: two contexts play ranks 0 and 1 of a
2-rank job, each builds its share of T3; rank 1's share is copied into rank 0's buffer (the byte movement
the NCCL all_gather performs across GPUs) and rank 0 must then produce exactly what an unsharded context
produces: all 162 counts of sampled quads and the rank-0 top-k."""
import numpy as np
import pytest

import datagen

pytestmark = pytest.mark.gpu


def _epi():
    import paper_conf_icpp_nobreiss22_b200 as epi
    return epi


@pytest.mark.parametrize("cfg,nsnp", [("C1", None), ("C2", 96), ("C5", 72)])
def test_sharded_t3_assembles_to_the_full_table(cfg, nsnp):
    import torch
    epi = _epi()
    d = datagen.make_config(cfg, n_snps=nsnp)
    rng = np.random.default_rng(7)
    quads = np.array([epi.pack_index(*sorted(rng.choice(d.n_snps, 4, replace=False))) for _ in range(300)],
                     dtype=np.uint64)
    with epi.Epi4(0, pipe="tc", rank=0, world=2) as ref:
        ref.load_genotypes(d.geno, d.phen)
        want_tab = ref.tables(quads)
        want_idx, want_k2 = ref.search(16)
    r0 = epi.Epi4(0, pipe="tc", rank=0, world=2, shard_t3=True)
    r1 = epi.Epi4(0, pipe="tc", rank=1, world=2, shard_t3=True)
    try:
        r0.load_genotypes(d.geno, d.phen)
        r1.load_genotypes(d.geno, d.phen)
        with pytest.raises(epi.Epi4Error):          # tables incomplete until the shares are gathered
            r0.search(16)
        full0, shard = r0.t3_device_view()
        full1, shard1 = r1.t3_device_view()
        assert shard == shard1 and full0.numel() == full1.numel() == 2 * shard
        full0[shard:2 * shard].copy_(full1[shard:2 * shard])
        torch.cuda.synchronize()
        epi.binding.epi4_t3_ready(r0.ctx)
        np.testing.assert_array_equal(r0.tables(quads), want_tab)
        idx, k2 = r0.search(16)
        np.testing.assert_array_equal(idx, want_idx)
        np.testing.assert_array_equal(k2, want_k2)
    finally:
        r0.close()
        r1.close()


def test_unsharded_context_refuses_shard_calls():
    epi = _epi()
    d = datagen.make_config("C1")
    with epi.Epi4(0, pipe="tc", rank=0, world=2) as e:
        e.load_genotypes(d.geno, d.phen)
        with pytest.raises(epi.Epi4Error):
            epi.binding.epi4_t3_shard(e.ctx)
        with pytest.raises(epi.Epi4Error):
            epi.binding.epi4_t3_ready(e.ctx)


@pytest.mark.parametrize("world", [2, 4])
def test_rank_partition_merges_to_the_single_rank_result(world):
    """SURVEY.md §4 T4 on one GPU: every rank of a `world`-rank plan searches only its LPT units; the
    deterministic merge of the per-rank top-k equals the 1-rank search (bit-identical keys)."""
    epi = _epi()
    d = datagen.make_config("C2", n_snps=96)
    with epi.Epi4(0, pipe="tc") as e:
        e.load_genotypes(d.geno, d.phen)
        want_idx, want_k2 = e.search(32)
    parts = []
    for r in range(world):
        with epi.Epi4(0, pipe="tc", rank=r, world=world) as e:
            e.load_genotypes(d.geno, d.phen)
            parts.append(e.search(32))
    idx, k2 = epi.merge_topk(parts, 32)
    np.testing.assert_array_equal(idx, want_idx)
    np.testing.assert_array_equal(k2, want_k2)


def test_multirank_path_on_one_gpu():
    """bench.py's N > 1 flow end to end (torchrun, 2 ranks on cuda:0 over gloo — NCCL refuses two ranks on
    one device): sharded T3 + all_gather, per-rank LPT units, all_gather + merge of the top-k."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--standalone", "--nproc-per-node", "2",
                        os.path.join(root, "tools", "multirank_one_gpu.py"), "--n-snps", "128"],
                       capture_output=True, text=True, timeout=600, cwd=root)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]
    assert "OK" in r.stdout


def test_multirank_nccl_on_two_gpus():
    """The same flow over NCCL with one rank per GPU (device-tensor all_gather of the T3 shares and of the top-k
    lists): needs >= 2 visible GPUs, skipped on a one-GPU box."""
    import os
    import subprocess
    import sys
    import torch
    if torch.cuda.device_count() < 2:
        pytest.skip("needs 2 GPUs (one rank per GPU over NCCL)")
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--standalone", "--nproc-per-node", "2",
                        os.path.join(root, "tools", "multirank_one_gpu.py"), "--backend", "nccl", "--n-snps", "160"],
                       capture_output=True, text=True, timeout=600, cwd=root)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-2000:]
    assert "OK" in r.stdout
