"""Slab-aware multi-GPU plan (PAPER.md:L128 phases the 3-way tables, L153-155 partitions the
work): with the windowed 3-way table each rank rebuilds the slabs FIRST(R) / FIRST(X) of the (R, X) groups it is
dealt, so the grouped plan must (1) cover every unit exactly once across ranks, (2) keep the ranks balanced and
(3) give each rank only ~1/world of the slab rebuilds (the ungrouped plan makes every rank rebuild nearly all)."""
import numpy as np
import pytest

from paper_conf_icpp_nobreiss22_b200 import binding

WINDOWED = binding.EPI4_FLAG_T3_WINDOWED


def _rebuilds(units):
    """Slab builds of a rank that walks its units in (R, X) order (api.cu epi4_search_units)."""
    groups = sorted({(int(w) * 128 // 128, int(x) // 128) for w, x in units})
    builds, slab_r, slab_x = 0, -1, -1
    for r, xr in groups:
        if r != slab_r:
            builds, slab_r = builds + 1, r
            if slab_x == slab_r:
                slab_x = -1
        if xr != r and xr != slab_x:
            builds, slab_x = builds + 1, xr
    return builds, len(groups)


@pytest.mark.parametrize("n,world", [(4096, 8), (4096, 4), (2048, 8), (300, 3)])
def test_grouped_plan_partitions_balances_and_localises_slabs(n, world):
    per_rank = [binding.epi4_plan_units_ex(n, r, world, WINDOWED) for r in range(world)]
    allu, allc = binding.epi4_plan_units(n, 0, 1)
    got = np.concatenate([u for u, _ in per_rank])
    assert len(got) == len(allu)
    key = lambda a: set(map(tuple, a.tolist()))
    assert key(got) == key(allu)                        # every unit once
    loads = np.array([c.sum() for _, c in per_rank])
    # makespan within 1 % of the mean in the windowed regime (N >= 2048; few, coarse units below)
    assert loads.max() / loads.mean() <= (1.01 if n >= 2048 else 1.05)
    total_groups = len({(int(w), int(x) // 128) for w, x in allu})
    builds = [_rebuilds(u)[0] for u, _ in per_rank]
    ungrouped = [_rebuilds(binding.epi4_plan_units(n, r, world)[0])[0] for r in range(world)]
    if n >= 2048:
        assert max(builds) <= 1.5 * total_groups / world + 16, (builds, total_groups)
        assert max(builds) * 2 < min(ungrouped), (builds, ungrouped)
