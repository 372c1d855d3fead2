"""Thin ctypes binding of libepi4 (include/epi4.h) — argument marshalling only.

Every function here has the name of the C entry point it wraps and does nothing but convert
arguments (numpy arrays, torch tensors or raw pointers) and raise on a negative return code.
All computation happens in libepi4's CUDA kernels.  There is deliberately no CPU fallback: if
libepi4.so is missing or fails to load, importing this module raises.
"""
from __future__ import annotations

import ctypes
import os
import re

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("EPI4_LIB") or os.path.join(HERE, "libepi4.so")   # EPI4_LIB: diagnostics builds only
HEADER = os.path.join(os.path.dirname(HERE), "include", "epi4.h")

EPI4_OK, EPI4_EINVAL, EPI4_ENOMEM, EPI4_ECUDA, EPI4_ESTATE, EPI4_ENODEV = 0, -1, -2, -3, -4, -5
EPI4_PIPE_TC, EPI4_PIPE_LOP3 = 0, 1
EPI4_PTR_HOST, EPI4_PTR_DEVICE = 0, 1
EPI4_FLAG_SHARD_T3 = 1
EPI4_FLAG_T3_WINDOWED = 2
EPI4_FLAG_TILE_N128 = 4
EPI4_FLAG_TILE_N224 = 8
EPI4_OBJ_K2, EPI4_OBJ_MI, EPI4_OBJ_CHI2 = 0, 1, 2
EPI4_MAX_TOPK = 1024
PIPES = {"tc": EPI4_PIPE_TC, "lop3": EPI4_PIPE_LOP3}


class Epi4Error(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"libepi4 error {code}: {msg}")
        self.code = code


class epi4_opts(ctypes.Structure):
    _fields_ = [("block", ctypes.c_int32), ("pipe", ctypes.c_int32), ("rank", ctypes.c_int32),
                ("world", ctypes.c_int32), ("grid", ctypes.c_int32), ("debug", ctypes.c_int32),
                ("flags", ctypes.c_int32), ("objective", ctypes.c_int32)]


class epi4_stats(ctypes.Structure):
    _fields_ = [("ms_pack", ctypes.c_double), ("ms_pop", ctypes.c_double), ("ms_quad", ctypes.c_double),
                ("ms_merge", ctypes.c_double), ("quads", ctypes.c_int64), ("tiles", ctypes.c_int64),
                ("launches", ctypes.c_int64), ("launches_load", ctypes.c_int64),
                ("executed_macs", ctypes.c_double), ("prof", ctypes.c_double * 8), ("tile_n", ctypes.c_int64)]

    def as_dict(self):
        d = {k: getattr(self, k) for k, _ in self._fields_}
        d["prof"] = list(self.prof)
        return d


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not built: run `python -c 'import __graft_entry__ as g; g.build()'`")
    lib = ctypes.CDLL(LIB_PATH)
    P, I32, I64 = ctypes.c_void_p, ctypes.c_int32, ctypes.c_int64
    sig = {
        "epi4_default_opts": (None, [ctypes.POINTER(epi4_opts)]),
        "epi4_create": (ctypes.c_int, [ctypes.POINTER(P), I32, ctypes.POINTER(epi4_opts)]),
        "epi4_destroy": (None, [P]),
        "epi4_set_stream": (ctypes.c_int, [P, P]),
        "epi4_load_bits": (ctypes.c_int, [P, P, P, I32, I64, I64, I32]),
        "epi4_pack_genotypes": (ctypes.c_int, [P, P, P, I32, I64, I32]),
        "epi4_get_bits": (ctypes.c_int, [P, P, P]),
        "epi4_search": (ctypes.c_int, [P, I32, P, P, P]),
        "epi4_search_units": (ctypes.c_int, [P, I64, I64, I32, P, P, P]),
        "epi4_search3": (ctypes.c_int, [P, I32, P, P, P]),
        "epi4_tables": (ctypes.c_int, [P, P, I64, P]),
        "epi4_set_dump": (ctypes.c_int, [P, P]),
        "epi4_set_sample": (ctypes.c_int, [P, I32, ctypes.c_uint64, I64]),
        "epi4_get_sample": (ctypes.c_int, [P, P, P, P, I64, ctypes.POINTER(I64)]),
        "epi4_t3_shard": (ctypes.c_int, [P, ctypes.POINTER(P), ctypes.POINTER(I64), ctypes.POINTER(I64)]),
        "epi4_t3_ready": (ctypes.c_int, [P]),
        "epi4_plan_count": (I64, [I32, I32, I32]),
        "epi4_plan_units": (ctypes.c_int, [I32, I32, I32, P, P]),
        "epi4_plan_count_ex": (I64, [I32, I32, I32, I32]),
        "epi4_plan_units_ex": (ctypes.c_int, [I32, I32, I32, I32, P, P]),
        "epi4_get_stats": (ctypes.c_int, [P, ctypes.POINTER(epi4_stats)]),
        "epi4_last_error": (ctypes.c_char_p, []),
        "epi4_version": (ctypes.c_char_p, []),
    }
    for name, (res, args) in sig.items():
        f = getattr(lib, name)
        f.restype = res
        f.argtypes = args
    return lib


_lib = _load()


def header_functions() -> list:
    """Names of the functions include/epi4.h declares."""
    txt = open(HEADER).read()
    txt = re.sub(r"/\*.*?\*/", "", txt, flags=re.S)
    return sorted(set(re.findall(r"\b(epi4_[a-z_0-9]+)\s*\(", txt)))


def _check(rc):
    if rc < 0:
        raise Epi4Error(rc, _lib.epi4_last_error().decode())
    return rc


def _ptr(x):
    """Raw address of a numpy array, a torch tensor, or an int pointer."""
    if x is None:
        return None
    if isinstance(x, int):
        return x
    if isinstance(x, np.ndarray):
        assert x.flags["C_CONTIGUOUS"]
        return x.ctypes.data
    if hasattr(x, "data_ptr"):
        assert x.is_contiguous()
        return x.data_ptr()
    raise TypeError(type(x))


def _kind(x):
    if hasattr(x, "is_cuda") and x.is_cuda:
        return EPI4_PTR_DEVICE
    return EPI4_PTR_HOST


def _dtype_name(x) -> str:
    """'uint8', 'uint32', ... for a numpy array or a torch tensor (None for raw pointers)."""
    if isinstance(x, np.ndarray):
        return x.dtype.name
    dt = getattr(x, "dtype", None)
    return None if dt is None else str(dt).replace("torch.", "")


def _require(x, name: str, dtype: str, shape: tuple):
    """Argument check for array inputs (raw int pointers are passed through unchecked): the C ABI reads
    `dtype` elements, so e.g. an int64 genotype array would be misread byte-wise."""
    if x is None or isinstance(x, int):
        return
    if _dtype_name(x) != dtype:
        raise TypeError(f"{name}: expected {dtype}, got {_dtype_name(x)}")
    if tuple(x.shape) != tuple(shape):
        raise ValueError(f"{name}: expected shape {tuple(shape)}, got {tuple(x.shape)}")
    contig = x.flags["C_CONTIGUOUS"] if isinstance(x, np.ndarray) else x.is_contiguous()
    if not contig:
        raise ValueError(f"{name}: must be C-contiguous")


def _same_kind(*xs) -> int:
    kinds = {_kind(x) for x in xs if x is not None and not isinstance(x, int)}
    if len(kinds) > 1:
        raise ValueError("all arrays of one call must be on the same side (all host or all device)")
    return kinds.pop() if kinds else EPI4_PTR_HOST


def epi4_default_opts() -> epi4_opts:
    o = epi4_opts()
    _lib.epi4_default_opts(ctypes.byref(o))
    return o


def epi4_create(cuda_device: int = 0, opts: epi4_opts | None = None) -> int:
    h = ctypes.c_void_p()
    _check(_lib.epi4_create(ctypes.byref(h), int(cuda_device), ctypes.byref(opts) if opts else None))
    return h.value


def epi4_destroy(ctx) -> None:
    _lib.epi4_destroy(ctx)


def epi4_set_stream(ctx, stream) -> None:
    _check(_lib.epi4_set_stream(ctx, stream))


def epi4_load_bits(ctx, planes_ctrl, planes_case, n_snps, n_controls, n_cases, ptr_kind=None) -> None:
    _require(planes_ctrl, "planes_ctrl", "uint32", (2 * int(n_snps), (int(n_controls) + 31) // 32))
    _require(planes_case, "planes_case", "uint32", (2 * int(n_snps), (int(n_cases) + 31) // 32))
    kind = _same_kind(planes_ctrl, planes_case) if ptr_kind is None else ptr_kind
    _check(_lib.epi4_load_bits(ctx, _ptr(planes_ctrl), _ptr(planes_case), int(n_snps), int(n_controls),
                               int(n_cases), kind))


def epi4_pack_genotypes(ctx, geno, phen, n_snps, n_samples, ptr_kind=None) -> None:
    _require(geno, "geno", "uint8", (int(n_snps), int(n_samples)))
    _require(phen, "phen", "uint8", (int(n_samples),))
    kind = _same_kind(geno, phen) if ptr_kind is None else ptr_kind
    _check(_lib.epi4_pack_genotypes(ctx, _ptr(geno), _ptr(phen), int(n_snps), int(n_samples), kind))


def epi4_get_bits(ctx, planes_ctrl: np.ndarray, planes_case: np.ndarray) -> None:
    _check(_lib.epi4_get_bits(ctx, _ptr(planes_ctrl), _ptr(planes_case)))


def epi4_search(ctx, top_k: int):
    q = np.zeros(top_k, dtype=np.uint64)
    k = np.zeros(top_k, dtype=np.float64)
    n = np.zeros(1, dtype=np.int32)
    _check(_lib.epi4_search(ctx, int(top_k), _ptr(q), _ptr(k), _ptr(n)))
    return q[: n[0]], k[: n[0]]


def epi4_search3(ctx, top_k: int):
    q = np.zeros(top_k, dtype=np.uint64)
    k = np.zeros(top_k, dtype=np.float64)
    n = np.zeros(1, dtype=np.int32)
    _check(_lib.epi4_search3(ctx, int(top_k), _ptr(q), _ptr(k), _ptr(n)))
    return q[: n[0]], k[: n[0]]


def epi4_search_units(ctx, unit_begin: int, unit_end: int, top_k: int):
    q = np.zeros(top_k, dtype=np.uint64)
    k = np.zeros(top_k, dtype=np.float64)
    n = np.zeros(1, dtype=np.int32)
    _check(_lib.epi4_search_units(ctx, int(unit_begin), int(unit_end), int(top_k), _ptr(q), _ptr(k), _ptr(n)))
    return q[: n[0]], k[: n[0]]


def epi4_tables(ctx, quads) -> np.ndarray:
    q = np.ascontiguousarray(np.asarray(quads, dtype=np.uint64).reshape(-1))
    out = np.zeros((q.size, 2, 81), dtype=np.uint32)
    _check(_lib.epi4_tables(ctx, _ptr(q), q.size, _ptr(out)))
    return out


def epi4_t3_shard(ctx):
    """(device address of the packed T3 buffer, bytes of one rank's share, total bytes)."""
    p, sb, tb = ctypes.c_void_p(), ctypes.c_int64(), ctypes.c_int64()
    _check(_lib.epi4_t3_shard(ctx, ctypes.byref(p), ctypes.byref(sb), ctypes.byref(tb)))
    return int(p.value or 0), int(sb.value), int(tb.value)


def epi4_t3_ready(ctx) -> None:
    _check(_lib.epi4_t3_ready(ctx))


def epi4_set_dump(ctx, counts_dev) -> None:
    _check(_lib.epi4_set_dump(ctx, _ptr(counts_dev)))


def epi4_set_sample(ctx, log2_rate: int, seed: int, capacity: int) -> None:
    _check(_lib.epi4_set_sample(ctx, int(log2_rate), ctypes.c_uint64(int(seed) & (2**64 - 1)), int(capacity)))


def epi4_get_sample(ctx, capacity: int):
    """(packed quads uint64[n], keys float64[n], counts uint32[n, 2, 81], total hits) of the last search."""
    q = np.zeros(max(capacity, 1), dtype=np.uint64)
    k = np.zeros(max(capacity, 1), dtype=np.float64)
    c = np.zeros((max(capacity, 1), 2, 81), dtype=np.uint32)
    n = ctypes.c_int64()
    _check(_lib.epi4_get_sample(ctx, _ptr(q), _ptr(k), _ptr(c), int(capacity), ctypes.byref(n)))
    m = min(int(n.value), int(capacity))
    return q[:m], k[:m], c[:m], int(n.value)


def epi4_plan_count(n_snps: int, rank: int = 0, world: int = 1) -> int:
    return _check(int(_lib.epi4_plan_count(int(n_snps), int(rank), int(world))))


def epi4_plan_units(n_snps: int, rank: int = 0, world: int = 1):
    cnt = epi4_plan_count(n_snps, rank, world)
    u = np.zeros((max(cnt, 1), 2), dtype=np.int32)
    c = np.zeros(max(cnt, 1), dtype=np.float64)
    _check(_lib.epi4_plan_units(int(n_snps), int(rank), int(world), _ptr(u), _ptr(c)))
    return u[:cnt], c[:cnt]


def epi4_plan_units_ex(n_snps: int, rank: int = 0, world: int = 1, flags: int = 0):
    cnt = _check(int(_lib.epi4_plan_count_ex(int(n_snps), int(rank), int(world), int(flags))))
    u = np.zeros((max(cnt, 1), 2), dtype=np.int32)
    c = np.zeros(max(cnt, 1), dtype=np.float64)
    _check(_lib.epi4_plan_units_ex(int(n_snps), int(rank), int(world), int(flags), _ptr(u), _ptr(c)))
    return u[:cnt], c[:cnt]


def epi4_get_stats(ctx) -> dict:
    s = epi4_stats()
    _check(_lib.epi4_get_stats(ctx, ctypes.byref(s)))
    return s.as_dict()


def epi4_last_error() -> str:
    return _lib.epi4_last_error().decode()


def epi4_version() -> str:
    return _lib.epi4_version().decode()
