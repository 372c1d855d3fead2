"""Host side of the verification-sample predicate of epi4_set_sample (include/epi4.h): which packed quad
indices the search kernels record.  Test helper only; it holds none of the method's arithmetic."""
import numpy as np

_C1 = np.uint64(0xBF58476D1CE4E5B9)
_C2 = np.uint64(0x94D049BB133111EB)


def mix64(x):
    x = np.asarray(x, dtype=np.uint64).copy()
    with np.errstate(over="ignore"):
        x ^= x >> np.uint64(30)
        x *= _C1
        x ^= x >> np.uint64(27)
        x *= _C2
        x ^= x >> np.uint64(31)
    return x


def sampled(packed, log2_rate: int, seed: int):
    mask = np.uint64((1 << log2_rate) - 1)
    return (mix64(np.asarray(packed, dtype=np.uint64) ^ np.uint64(seed)) & mask) == 0


def pack(q):
    q = np.asarray(q, dtype=np.uint64).reshape(-1, 4)
    return (q[:, 0] << np.uint64(48)) | (q[:, 1] << np.uint64(32)) | (q[:, 2] << np.uint64(16)) | q[:, 3]


def unpack(idx):
    idx = np.asarray(idx, dtype=np.uint64)
    return np.stack([(idx >> np.uint64(s)) & np.uint64(0xFFFF) for s in (48, 32, 16, 0)], axis=1).astype(np.int64)


def rate_for(n_quads: int, target: int) -> int:
    """log2 sampling rate giving about `target` hits out of n_quads."""
    r = 0
    while n_quads / (1 << (r + 1)) >= target:
        r += 1
    return r
