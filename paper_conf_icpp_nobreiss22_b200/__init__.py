"""B200-native exhaustive fourth-order K2 epistasis search (Epi4Tensor's hot path, PAPER.md).

The search runs in libepi4 (CUDA kernels for sm_100a behind the C ABI of include/epi4.h); this
package is the thin Python layer: the ctypes binding (``binding``), a small object wrapper and the
multi-GPU glue (one process per GPU; the per-rank top-k lists are all-gathered over NCCL/NVLink and
merged deterministically — SURVEY.md §8(e)).
"""
from __future__ import annotations

import numpy as np

from . import binding
from .binding import Epi4Error, epi4_last_error, epi4_version  # noqa: F401

__all__ = ["Epi4", "merge_topk", "search_distributed", "allgather_shares", "pack_index", "unpack_index", "binding", "Epi4Error"]


def pack_index(i, j, k, l) -> int:
    """four 16-bit SNP indices in one 64-bit word."""
    return (int(i) << 48) | (int(j) << 32) | (int(k) << 16) | int(l)


def unpack_index(idx) -> tuple:
    idx = int(idx)
    return ((idx >> 48) & 0xFFFF, (idx >> 32) & 0xFFFF, (idx >> 16) & 0xFFFF, idx & 0xFFFF)


class Epi4:
    """One search context on one GPU (one per rank)."""

    def __init__(self, device: int = 0, pipe: str = "tc", rank: int = 0, world: int = 1, grid: int = 0,
                 debug: int = 0, shard_t3: bool = False, t3_windowed: bool = False, objective: str = "k2",
                 tile: int | None = None):
        o = binding.epi4_default_opts()
        o.pipe = binding.PIPES[pipe]
        o.rank, o.world, o.grid = int(rank), int(world), int(grid)
        o.debug = int(debug)           # diagnostics only: disables warp roles, results invalid
        o.flags = (binding.EPI4_FLAG_SHARD_T3 if shard_t3 else 0) | (binding.EPI4_FLAG_T3_WINDOWED if t3_windowed else 0)
        if tile not in (None, 128, 224):
            raise ValueError("tile must be None (chosen by the load), 128 or 224")
        o.flags |= {None: 0, 128: binding.EPI4_FLAG_TILE_N128, 224: binding.EPI4_FLAG_TILE_N224}[tile]
        o.objective = {"k2": binding.EPI4_OBJ_K2, "mi": binding.EPI4_OBJ_MI,
                       "chi2": binding.EPI4_OBJ_CHI2}[objective]
        self.shard_t3 = bool(shard_t3) and int(world) > 1
        self.pipe, self.rank, self.world = pipe, int(rank), int(world)
        self.ctx = binding.epi4_create(device, o)

    def close(self):
        if getattr(self, "ctx", None):
            binding.epi4_destroy(self.ctx)
            self.ctx = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def __enter__(self):
        return self

    def __exit__(self, *a):
        self.close()

    def set_stream(self, stream):
        binding.epi4_set_stream(self.ctx, stream)

    def load_genotypes(self, geno, phen):
        """Byte genotypes N x M (SNP-major, {0,1,2}) + phenotypes M; host (numpy) or device (torch)."""
        if getattr(geno, "ndim", None) != 2:
            raise ValueError("geno must be a 2-D N x M array")
        n, m = geno.shape
        binding.epi4_pack_genotypes(self.ctx, geno, phen, n, m)

    def load_bits(self, planes_ctrl, planes_case, n_snps, n_controls, n_cases):
        binding.epi4_load_bits(self.ctx, planes_ctrl, planes_case, n_snps, n_controls, n_cases)

    def search(self, top_k: int = 1):
        return binding.epi4_search(self.ctx, top_k)

    def search3(self, top_k: int = 1):
        """Third-order search: (packed i<<48|j<<32|k<<16, K2 over 27 cells)."""
        return binding.epi4_search3(self.ctx, top_k)

    def search_units(self, unit_begin: int, unit_end: int, top_k: int = 1):
        return binding.epi4_search_units(self.ctx, unit_begin, unit_end, top_k)

    def t3_device_view(self):
        """(full uint8 device tensor over the packed T3 buffer, share size in bytes) — sharded T3 only."""
        import torch
        ptr, shard, total = binding.epi4_t3_shard(self.ctx)
        return torch.as_tensor(_CudaBuffer(ptr, total), device="cuda"), shard

    def gather_t3(self, group=None, stream=None):
        """Sharded T3: all-gather the ranks' equal-size shares of the 3-way table over
        torch.distributed (NCCL over NVLink on GPUs), then release the context for searching."""
        import torch
        full, shard = self.t3_device_view()
        allgather_shares(full, shard, group)
        torch.cuda.current_stream().synchronize()
        binding.epi4_t3_ready(self.ctx)

    def set_sample(self, log2_rate: int, seed: int = 0, capacity: int = 1 << 16):
        """Verification sample of the next searches (epi4_set_sample); capacity 0 disables."""
        binding.epi4_set_sample(self.ctx, log2_rate, seed, capacity)
        self._samp_cap = int(capacity)

    def get_sample(self):
        """(packed quads, keys, counts [n, 2, 81], total hits) recorded by the last search."""
        return binding.epi4_get_sample(self.ctx, getattr(self, "_samp_cap", 0))

    def tables(self, quads):
        return binding.epi4_tables(self.ctx, quads)

    def stats(self) -> dict:
        return binding.epi4_get_stats(self.ctx)


class _CudaBuffer:
    """A raw device allocation exposed through __cuda_array_interface__ (uint8), for torch.as_tensor."""

    def __init__(self, ptr: int, nbytes: int):
        self.__cuda_array_interface__ = {"shape": (int(nbytes),), "typestr": "|u1", "data": (int(ptr), False),
                                         "version": 3, "strides": None}


def allgather_shares(full, shard: int, group=None):
    """In-place assembly of equal-size shares: rank r's bytes live in full[r*shard:(r+1)*shard]; after the
    call every rank holds all of them (one all_gather of `shard` bytes per rank; NCCL or gloo)."""
    import torch.distributed as dist
    r = dist.get_rank(group)
    if full.is_cuda and dist.get_backend(group) != "nccl":   # gloo (tests, one-GPU runs): stage through the host
        host = full.cpu()
        allgather_shares(host, shard, group)
        full.copy_(host)
        return full
    mine = full[r * shard:(r + 1) * shard].clone()
    dist.all_gather_into_tensor(full, mine, group=group)
    return full


def merge_topk(parts, top_k: int):
    """Deterministic merge of (idx uint64[], k2 float64[]) lists by the (K2, index) key."""
    idx = np.concatenate([np.asarray(p[0], dtype=np.uint64) for p in parts]) if parts else np.zeros(0, np.uint64)
    k2 = np.concatenate([np.asarray(p[1], dtype=np.float64) for p in parts]) if parts else np.zeros(0)
    order = np.lexsort((idx, k2))[:top_k]
    return idx[order], k2[order]


def search_distributed(local_search, top_k: int, group=None, device=None):
    """Run ``local_search(top_k)`` on every rank, all-gather the per-rank lists and merge them
    (the single collective of the search).  Works with NCCL (device tensors) and
    gloo (CPU tensors)."""
    import torch
    import torch.distributed as dist

    idx, k2 = local_search(top_k)
    world = dist.get_world_size(group)
    dev = device if device is not None else ("cuda" if dist.get_backend(group) == "nccl" else "cpu")
    buf = torch.full((top_k, 2), float("inf"), dtype=torch.float64)
    n = len(idx)
    buf[:n, 0] = torch.from_numpy(np.asarray(k2, dtype=np.float64))
    buf[:n, 1] = torch.from_numpy(np.asarray(idx, dtype=np.uint64).view(np.float64))   # bit-cast
    cnt = torch.tensor([n], dtype=torch.int64)
    buf, cnt = buf.to(dev), cnt.to(dev)
    bufs = [torch.empty_like(buf) for _ in range(world)]
    cnts = [torch.empty_like(cnt) for _ in range(world)]
    dist.all_gather(bufs, buf, group=group)
    dist.all_gather(cnts, cnt, group=group)
    parts = []
    for b, c in zip(bufs, cnts):
        b = b.cpu().numpy()
        c = int(c.item())
        parts.append((b[:c, 1].copy().view(np.uint64), b[:c, 0].copy()))
    return merge_topk(parts, top_k)
