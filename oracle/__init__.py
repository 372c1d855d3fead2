"""CPU oracle for the fourth-order K2 epistasis search — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  It shares no code with the CUDA
path (``paper_conf_icpp_nobreiss22_b200``) and neither imports the other; the only
shared module is the input generator ``datagen``.

The arithmetic lives in ``epi4_oracle.c`` (plain C, per-quad per-sample loops, K2 in
double via glibc lgamma); see its header for the PAPER.md passages it follows and the
DESIGN.md readings.  This file is argument marshalling via ctypes plus a few small
numpy helpers used by the pins (brute-force 3-/2-way tables written separately from
the C code).
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "epi4_oracle.c")
_LIB = os.path.join(_HERE, "libepi4_oracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile the oracle shared library (gcc, OpenMP, no fast-math, no FP contraction)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        cmd = ["gcc", "-O3", "-std=c11", "-fopenmp", "-fPIC", "-shared", "-fno-fast-math",
               "-ffp-contract=off", "-o", _LIB + ".tmp", _SRC, "-lm"]
        subprocess.run(cmd, check=True)
        os.replace(_LIB + ".tmp", _LIB)
    return _LIB


def _load():
    global _lib
    if _lib is None:
        build()
        lib = ctypes.CDLL(_LIB)
        P = ctypes.c_void_p
        lib.oracle_k2.restype = ctypes.c_double
        lib.oracle_k2.argtypes = [P]
        lib.oracle_pack.restype = ctypes.c_uint64
        lib.oracle_pack.argtypes = [ctypes.c_int32] * 4
        lib.oracle_tables.restype = ctypes.c_int
        lib.oracle_tables.argtypes = [P, P, ctypes.c_int32, ctypes.c_int64, P, ctypes.c_int64, P, ctypes.c_int32]
        lib.oracle_score.restype = ctypes.c_int
        lib.oracle_score.argtypes = [P, P, ctypes.c_int32, ctypes.c_int64, P, ctypes.c_int64, P, ctypes.c_int32]
        lib.oracle_search.restype = ctypes.c_int
        lib.oracle_search.argtypes = [P, P, ctypes.c_int32, ctypes.c_int64, ctypes.c_int32, P, P, P, ctypes.c_int32]
        lib.oracle_tables3.restype = ctypes.c_int
        lib.oracle_tables3.argtypes = [P, P, ctypes.c_int32, ctypes.c_int64, P, ctypes.c_int64, P]
        lib.oracle_search3.restype = ctypes.c_int
        lib.oracle_search3.argtypes = [P, P, ctypes.c_int32, ctypes.c_int64, ctypes.c_int32, P, P, P, ctypes.c_int32]
        lib.oracle_mi.restype = ctypes.c_double
        lib.oracle_mi.argtypes = [P]
        lib.oracle_search_mi.restype = ctypes.c_int
        lib.oracle_search_mi.argtypes = [P, P, ctypes.c_int32, ctypes.c_int64, ctypes.c_int32, P, P, P]
        lib.oracle_chi2.restype = ctypes.c_double
        lib.oracle_chi2.argtypes = [P]
        lib.oracle_search_chi2.restype = ctypes.c_int
        lib.oracle_search_chi2.argtypes = [P, P, ctypes.c_int32, ctypes.c_int64, ctypes.c_int32, P, P, P]
        lib.oracle_score3_obj.restype = ctypes.c_double
        lib.oracle_score3_obj.argtypes = [P, ctypes.c_int32]
        lib.oracle_search3_obj.restype = ctypes.c_int
        lib.oracle_search3_obj.argtypes = [P, P, ctypes.c_int32, ctypes.c_int64, ctypes.c_int32, ctypes.c_int32, P, P, P]
        lib.oracle_max_threads.restype = ctypes.c_int32
        lib.oracle_max_threads.argtypes = [ctypes.c_int32]
        _lib = lib
    return _lib


def _ptr(a: np.ndarray):
    return a.ctypes.data_as(ctypes.c_void_p)


def _prep(geno, phen):
    geno = np.ascontiguousarray(geno, dtype=np.uint8)
    phen = np.ascontiguousarray(phen, dtype=np.uint8)
    assert geno.ndim == 2 and phen.shape == (geno.shape[1],)
    return geno, phen


def pack_index(i, j, k, l) -> int:
    """PAPER.md:L145 packed quad index i<<48 | j<<32 | k<<16 | l."""
    return int(_load().oracle_pack(int(i), int(j), int(k), int(l)))


def unpack_index(idx) -> tuple:
    idx = int(idx)
    return ((idx >> 48) & 0xFFFF, (idx >> 32) & 0xFFFF, (idx >> 16) & 0xFFFF, idx & 0xFFFF)


def k2(table) -> float:
    """K2 of a 2 x 81 table (row 0 controls, row 1 cases)."""
    t = np.ascontiguousarray(np.asarray(table, dtype=np.uint32).reshape(2, 81))
    return float(_load().oracle_k2(_ptr(t)))


def tables(geno, phen, quads, n_threads: int = 0) -> np.ndarray:
    """Per-sample brute-force 2 x 81 tables for the given quads -> uint32 [nq, 2, 81]."""
    geno, phen = _prep(geno, phen)
    q = np.ascontiguousarray(np.asarray(quads, dtype=np.int32).reshape(-1, 4))
    out = np.zeros((q.shape[0], 2, 81), dtype=np.uint32)
    rc = _load().oracle_tables(_ptr(geno), _ptr(phen), geno.shape[0], geno.shape[1], _ptr(q),
                               q.shape[0], _ptr(out), n_threads)
    if rc:
        raise ValueError(f"oracle_tables failed: {rc}")
    return out


def score(geno, phen, quads, n_threads: int = 0) -> np.ndarray:
    """K2 (double) for the given quads."""
    geno, phen = _prep(geno, phen)
    q = np.ascontiguousarray(np.asarray(quads, dtype=np.int32).reshape(-1, 4))
    out = np.zeros(q.shape[0], dtype=np.float64)
    rc = _load().oracle_score(_ptr(geno), _ptr(phen), geno.shape[0], geno.shape[1], _ptr(q),
                              q.shape[0], _ptr(out), n_threads)
    if rc:
        raise ValueError(f"oracle_score failed: {rc}")
    return out


def search(geno, phen, top_k: int = 1, n_snps: int | None = None, n_threads: int = 0):
    """Exhaustive search over all quads of SNPs [0, n_snps) -> (packed idx uint64[k], K2 float64[k])."""
    geno, phen = _prep(geno, phen)
    n = geno.shape[0] if n_snps is None else int(n_snps)
    geno = np.ascontiguousarray(geno[:n])
    idx = np.zeros(top_k, dtype=np.uint64)
    k2v = np.zeros(top_k, dtype=np.float64)
    nout = np.zeros(1, dtype=np.int32)
    rc = _load().oracle_search(_ptr(geno), _ptr(phen), n, geno.shape[1], int(top_k), _ptr(idx),
                               _ptr(k2v), _ptr(nout), n_threads)
    if rc:
        raise ValueError(f"oracle_search failed: {rc}")
    return idx[: nout[0]], k2v[: nout[0]]


def mi(table) -> float:
    """M * I (mutual information of the 81-cell genotype and the phenotype, nats) of a 2 x 81 table."""
    t = np.ascontiguousarray(np.asarray(table, dtype=np.uint32).reshape(2, 81))
    return float(_load().oracle_mi(_ptr(t)))


def search_mi(geno, phen, top_k: int = 1, n_snps: int | None = None):
    """Exhaustive search ranked by mutual information -> (packed idx, key = -M*I),
    the top_k smallest keys ascending (single-threaded: for small test problems)."""
    geno, phen = _prep(geno, phen)
    n = geno.shape[0] if n_snps is None else int(n_snps)
    geno = np.ascontiguousarray(geno[:n])
    idx = np.zeros(top_k, dtype=np.uint64)
    key = np.zeros(top_k, dtype=np.float64)
    nout = np.zeros(1, dtype=np.int32)
    rc = _load().oracle_search_mi(_ptr(geno), _ptr(phen), n, geno.shape[1], int(top_k), _ptr(idx), _ptr(key),
                                  _ptr(nout))
    if rc:
        raise ValueError(f"oracle_search_mi failed: {rc}")
    return idx[: nout[0]], key[: nout[0]]


def chi2(table) -> float:
    """Pearson chi-square (no continuity correction) of a 2 x 81 table over its non-empty genotype cells."""
    t = np.ascontiguousarray(np.asarray(table, dtype=np.uint32).reshape(2, 81))
    return float(_load().oracle_chi2(_ptr(t)))


def search_chi2(geno, phen, top_k: int = 1, n_snps: int | None = None):
    """Exhaustive search ranked by Pearson chi-square -> (packed idx, key = -X^2),
    the top_k smallest keys ascending (single-threaded: for small test problems)."""
    geno, phen = _prep(geno, phen)
    n = geno.shape[0] if n_snps is None else int(n_snps)
    geno = np.ascontiguousarray(geno[:n])
    idx = np.zeros(top_k, dtype=np.uint64)
    key = np.zeros(top_k, dtype=np.float64)
    nout = np.zeros(1, dtype=np.int32)
    rc = _load().oracle_search_chi2(_ptr(geno), _ptr(phen), n, geno.shape[1], int(top_k), _ptr(idx), _ptr(key),
                                    _ptr(nout))
    if rc:
        raise ValueError(f"oracle_search_chi2 failed: {rc}")
    return idx[: nout[0]], key[: nout[0]]


def tables3(geno, phen, triples) -> np.ndarray:
    """Per-sample brute-force 2 x 27 tables (cell 9a + 3b + c) of the given triples -> uint32 [nt, 2, 27]."""
    geno, phen = _prep(geno, phen)
    t = np.ascontiguousarray(np.asarray(triples, dtype=np.int32).reshape(-1, 3))
    out = np.zeros((t.shape[0], 2, 27), dtype=np.uint32)
    rc = _load().oracle_tables3(_ptr(geno), _ptr(phen), geno.shape[0], geno.shape[1], _ptr(t), t.shape[0], _ptr(out))
    if rc:
        raise ValueError(f"oracle_tables3 failed: {rc}")
    return out


def search3(geno, phen, top_k: int = 1, n_snps: int | None = None, n_threads: int = 0):
    """Exhaustive third-order search over all triples of SNPs [0, n_snps) -> (packed idx i<<48|j<<32|k<<16,
    K2 over 27 cells), the top_k smallest (K2, idx) keys ascending."""
    geno, phen = _prep(geno, phen)
    n = geno.shape[0] if n_snps is None else int(n_snps)
    geno = np.ascontiguousarray(geno[:n])
    idx = np.zeros(top_k, dtype=np.uint64)
    k2v = np.zeros(top_k, dtype=np.float64)
    nout = np.zeros(1, dtype=np.int32)
    rc = _load().oracle_search3(_ptr(geno), _ptr(phen), n, geno.shape[1], int(top_k), _ptr(idx), _ptr(k2v),
                                _ptr(nout), n_threads)
    if rc:
        raise ValueError(f"oracle_search3 failed: {rc}")
    return idx[: nout[0]], k2v[: nout[0]]


_OBJ3 = {"mi": 1, "chi2": 2}


def score3(table, objective: str) -> float:
    """M * I ("mi") or Pearson X^2 ("chi2") of a 2 x 27 triple table."""
    t = np.ascontiguousarray(np.asarray(table, dtype=np.uint32).reshape(2, 27))
    return float(_load().oracle_score3_obj(_ptr(t), _OBJ3[objective]))


def search3_obj(geno, phen, objective: str, top_k: int = 1, n_snps: int | None = None):
    """Exhaustive third-order search ranked by "mi" or "chi2" (SURVEY.md §8(f) NEXT-3 x NEXT-4) -> (packed idx,
    key = -score), the top_k smallest keys ascending (single-threaded: for small test problems)."""
    geno, phen = _prep(geno, phen)
    n = geno.shape[0] if n_snps is None else int(n_snps)
    geno = np.ascontiguousarray(geno[:n])
    idx = np.zeros(top_k, dtype=np.uint64)
    key = np.zeros(top_k, dtype=np.float64)
    nout = np.zeros(1, dtype=np.int32)
    rc = _load().oracle_search3_obj(_ptr(geno), _ptr(phen), n, geno.shape[1], int(top_k), _OBJ3[objective],
                                    _ptr(idx), _ptr(key), _ptr(nout))
    if rc:
        raise ValueError(f"oracle_search3_obj failed: {rc}")
    return idx[: nout[0]], key[: nout[0]]


def max_threads(n_threads: int = 0) -> int:
    return int(_load().oracle_max_threads(n_threads))
