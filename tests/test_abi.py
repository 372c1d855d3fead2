"""CPU tests of the C ABI library: it loads, exports every symbol include/epi4.h declares, reports
errors through return codes (no GPU needed), and the host-side plan is a correct, balanced partition."""
import ctypes
import itertools

import numpy as np
import pytest

import paper_conf_icpp_nobreiss22_b200 as epi
from paper_conf_icpp_nobreiss22_b200 import binding


def test_library_exports_every_header_symbol():
    names = binding.header_functions()
    assert len(names) >= 15
    lib = ctypes.CDLL(binding.LIB_PATH)
    for n in names:
        assert hasattr(lib, n), n
    assert "sm_100a" in epi.epi4_version()


def test_library_is_sm100a_only():
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", binding.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out
    for other in ("sm_80", "sm_90", "sm_89"):
        assert other + "." not in out


def test_create_without_device_fails_cleanly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    with pytest.raises(binding.Epi4Error) as ei:
        binding.epi4_create(0)
    assert ei.value.code == binding.EPI4_ENODEV
    assert "device" in binding.epi4_last_error()


def test_plan_rejects_bad_arguments():
    with pytest.raises(binding.Epi4Error):
        binding.epi4_plan_count(3, 0, 1)
    with pytest.raises(binding.Epi4Error):
        binding.epi4_plan_count(40, 2, 2)


def _quads_of_unit(n, wb, x):
    for w in range(128 * wb, min(128 * wb + 128, x)):
        for y in range(x + 1, n):
            for z in range(y + 1, n):
                yield (w, x, y, z)


@pytest.mark.parametrize("n", [4, 5, 33, 40, 70])
def test_plan_covers_every_quad_exactly_once(n):
    units, cost = binding.epi4_plan_units(n, 0, 1)
    seen = []
    for wb, x in units:
        seen.extend(_quads_of_unit(n, int(wb), int(x)))
    assert len(seen) == len(set(seen))
    assert set(seen) == set(itertools.combinations(range(n), 4))
    assert (np.diff(cost) <= 0).all()          # longest first


@pytest.mark.parametrize("n,world", [(40, 2), (70, 3), (512, 8), (2048, 8)])
def test_plan_partition_across_ranks(n, world):
    allu, allc = binding.epi4_plan_units(n, 0, 1)
    parts = [binding.epi4_plan_units(n, r, world) for r in range(world)]
    got = sorted((int(a), int(b)) for u, _ in parts for a, b in u)
    assert got == sorted((int(a), int(b)) for a, b in allu)
    loads = np.array([c.sum() for _, c in parts])
    assert loads.sum() == pytest.approx(allc.sum())
    if n >= 512:
        assert loads.max() / loads.mean() < 1.01    # LPT makespan ~1.000


def test_plan_is_deterministic():
    a = binding.epi4_plan_units(512, 3, 8)
    b = binding.epi4_plan_units(512, 3, 8)
    np.testing.assert_array_equal(a[0], b[0])


def test_merge_topk_orders_by_key_then_index():
    parts = [(np.array([5, 3], np.uint64), np.array([1.0, 2.0])),
             (np.array([2, 9, 4], np.uint64), np.array([1.0, 0.5, 2.0]))]
    idx, k2 = epi.merge_topk(parts, 4)
    assert list(idx) == [9, 2, 5, 3]
    assert list(k2) == [0.5, 1.0, 1.0, 2.0]


def test_binding_constants_match_the_header():
    """Every EPI4_* integer #define in include/epi4.h that the binding mirrors has the same value."""
    import os
    import re
    hdr = open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "include", "epi4.h")).read()
    defs = {m.group(1): int(m.group(2), 0) for m in re.finditer(r"#define\s+(EPI4_\w+)\s+\(?(-?(?:0x)?[0-9A-Fa-f]+)\)?", hdr)}
    for name in ("EPI4_OBJ_K2", "EPI4_OBJ_MI", "EPI4_OBJ_CHI2", "EPI4_FLAG_SHARD_T3", "EPI4_FLAG_T3_WINDOWED",
                 "EPI4_FLAG_TILE_N128", "EPI4_FLAG_TILE_N224",
                 "EPI4_EINVAL", "EPI4_ENODEV", "EPI4_PIPE_TC", "EPI4_PIPE_LOP3"):
        assert name in defs, name
        assert getattr(binding, name) == defs[name], name


def test_tile_option_is_validated_before_any_device_call():
    """Epi4(tile=...) accepts only None / 128 / 224 (EPI4_FLAG_TILE_*); anything else fails in the binding,
    before a context is created."""
    import pytest
    import paper_conf_icpp_nobreiss22_b200 as epi
    with pytest.raises(ValueError):
        epi.Epi4(0, tile=160)
