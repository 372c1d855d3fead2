"""Multi-process (gloo, world_size 2) test of the N>1 host path: the static LPT plan splits the quad
space across ranks, each rank produces its local top-k, one all_gather + deterministic merge gives the
global answer.  The per-rank local search is stood in for by the oracle restricted to the rank's units
(no GPU here); the product pieces under test are epi4_plan_units and search_distributed."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import datagen
import oracle


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, top_k, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_icpp_nobreiss22_b200 as epi
        from paper_conf_icpp_nobreiss22_b200 import binding
        d = datagen.make_config("C1")
        n = d.n_snps
        units, _ = binding.epi4_plan_units(n, rank, world)
        quads = []
        for wb, x in units:
            for w in range(128 * wb, min(128 * wb + 128, x)):
                for y in range(x + 1, n):
                    for z in range(y + 1, n):
                        quads.append((w, int(x), y, z))
        quads = np.array(quads, dtype=np.int32).reshape(-1, 4)

        def local(k):
            k2 = oracle.score(d.geno, d.phen, quads, n_threads=1)
            idx = np.array([oracle.pack_index(*qq) for qq in quads], dtype=np.uint64)
            order = np.lexsort((idx, k2))[:k]
            return idx[order], k2[order]

        idx, k2 = epi.search_distributed(local, top_k)
        q.put((rank, len(quads), idx.tolist(), k2.tolist()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_two_rank_search_matches_single_process(world):
    top_k = 10
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, top_k, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    d = datagen.make_config("C1")
    ref_idx, ref_k2 = oracle.search(d.geno, d.phen, top_k=top_k)
    assert sum(r[1] for r in res) == 91390          # the ranks' units partition C(40,4)
    for _, _, idx, k2 in res:                        # every rank holds the same merged answer
        assert idx == [int(v) for v in ref_idx]
        assert k2 == [float(v) for v in ref_k2]


def _shard_worker(rank, world, port, shard, q):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_icpp_nobreiss22_b200 as epi
        full = torch.zeros(world * shard, dtype=torch.uint8)
        full[rank * shard:(rank + 1) * shard] = torch.arange(shard, dtype=torch.int64).remainder(251).to(torch.uint8) + rank
        epi.allgather_shares(full, shard)
        q.put((rank, full.numpy().tobytes()))
    finally:
        dist.destroy_process_group()


def test_sharded_table_allgather_assembles_every_share():
    """The N > 1 sharded-T3 exchange (bench.py, Epi4.gather_t3): equal-size shares, in-place assembly."""
    world, shard = 2, 1000
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_shard_worker, args=(r, world, port, shard, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    want = np.concatenate([(np.arange(shard) % 251 + r).astype(np.uint8) for r in range(world)]).tobytes()
    assert res[0] == want and res[1] == want
