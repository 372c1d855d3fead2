"""Seeded synthetic case/control genotype generator (shared INPUT module).

This module is the only code shared by the oracle (``oracle/``) and the CUDA
path (``paper_conf_icpp_nobreiss22_b200/``).  It holds none of the method's
arithmetic: it draws genotypes and phenotype labels and nothing else (no
counting, no packing, no scoring).

Recipe ("synthetic (i.e. randomly generated)"
datasets with half cases / half controls):

* genotype codes 0 = AA (homozygous major), 1 = Aa, 2 = aa;
* per SNP a minor-allele frequency q ~ U(0.05, 0.5) and i.i.d. Hardy-Weinberg
  genotypes with probabilities (1-q)^2, 2q(1-q), q^2;
* exact class sizes: ``n_cases`` samples have phenotype 1, ``n_controls``
  phenotype 0, in a seeded random order (so the pack step must split them);
* an optional planted 4-way interaction: a quad whose case probability is
  0.9 when the number of heterozygous genotypes in the quad is odd and 0.1
  otherwise.  The quad's genotypes are drawn from their
  exact conditional distribution given each sample's phenotype
  (P(g | p) ∝ P_HWE(g) · P(p | g)), which is what rejection sampling
  conditional on the phenotype converges to, and keeps class sizes exact;
* ``uniform=True`` draws every genotype uniformly from {0,1,2} (sensitivity
  run).

Everything is drawn from one ``numpy.random.Generator(PCG64(seed))``.
"""
from __future__ import annotations

import dataclasses
import itertools

import numpy as np

__all__ = ["Dataset", "CONFIGS", "make_dataset", "make_config", "planted_quad_for",
           "hand_dataset"]


@dataclasses.dataclass
class Dataset:
    geno: np.ndarray        # uint8 [N, M], SNP-major, values in {0,1,2}
    phen: np.ndarray        # uint8 [M], 0 = control, 1 = case
    n_controls: int
    n_cases: int
    planted: tuple | None   # planted quad (i<j<k<l) or None
    seed: int
    name: str = ""

    @property
    def n_snps(self) -> int:
        return int(self.geno.shape[0])

    @property
    def n_samples(self) -> int:
        return int(self.geno.shape[1])


# BASELINE.json "configs" (N = SNPs, M = samples; repo naming).
CONFIGS = {
    "C1": dict(n_snps=40, n_controls=256, n_cases=256, index=0),
    "C2": dict(n_snps=512, n_controls=8192, n_cases=8192, index=1),
    "C3": dict(n_snps=2048, n_controls=16384, n_cases=16384, index=2),
    "C4": dict(n_snps=4096, n_controls=32768, n_cases=32768, index=3),
    # M = 100003, 30/70 split: n1 = round(0.3 * 100003) = 30001 cases
    "C5": dict(n_snps=1024, n_controls=70002, n_cases=30001, index=4),
}


def planted_quad_for(n_snps: int) -> tuple:
    """Planted quad position."""
    if n_snps == 40:
        return (3, 11, 22, 35)
    n = n_snps
    return (5, n // 4 + 7, n // 2 + 13, 3 * n // 4 + 29)


def _hwe_probs(q: np.ndarray) -> np.ndarray:
    return np.stack([(1 - q) ** 2, 2 * q * (1 - q), q ** 2], axis=-1)


def make_dataset(n_snps: int, n_controls: int, n_cases: int, seed: int,
                 planted: tuple | None = None, uniform: bool = False,
                 penetrance=(0.1, 0.9), maf_range=(0.05, 0.5), name: str = "") -> Dataset:
    rng = np.random.Generator(np.random.PCG64(seed))
    n, m = int(n_snps), int(n_controls) + int(n_cases)
    phen = np.zeros(m, dtype=np.uint8)
    phen[:n_cases] = 1
    rng.shuffle(phen)
    if uniform:
        geno = rng.integers(0, 3, size=(n, m), dtype=np.uint8)
        q = None
    else:
        q = rng.uniform(maf_range[0], maf_range[1], size=n)
        p0 = (1 - q) ** 2
        p01 = p0 + 2 * q * (1 - q)
        geno = np.empty((n, m), dtype=np.uint8)
        chunk = max(1, (1 << 24) // max(m, 1))
        for s in range(0, n, chunk):
            e = min(n, s + chunk)
            u = rng.random((e - s, m))
            geno[s:e] = (u >= p0[s:e, None]).astype(np.uint8) + (u >= p01[s:e, None]).astype(np.uint8)
    if planted is not None:
        quad = tuple(int(v) for v in planted)
        assert len(quad) == 4 and list(quad) == sorted(set(quad)) and quad[-1] < n
        if q is None:
            pg = np.full((4, 3), 1.0 / 3.0)
        else:
            pg = _hwe_probs(q[list(quad)])
        cells = np.array(list(itertools.product(range(3), repeat=4)), dtype=np.uint8)  # 81 x 4
        prior = np.prod(pg[np.arange(4)[None, :], cells], axis=1)
        nhet = (cells == 1).sum(axis=1)
        p_case = np.where(nhet % 2 == 1, penetrance[1], penetrance[0])
        for pv, like in ((1, p_case), (0, 1.0 - p_case)):
            post = prior * like
            post = post / post.sum()
            idx = np.nonzero(phen == pv)[0]
            draw = rng.choice(81, size=idx.size, p=post)
            geno[np.array(quad)[:, None], idx[None, :]] = cells[draw].T
    return Dataset(geno=geno, phen=phen, n_controls=int(n_controls), n_cases=int(n_cases),
                   planted=None if planted is None else tuple(planted), seed=seed, name=name)


def make_config(name: str, planted: bool = True, uniform: bool = False, seed: int | None = None,
                n_snps: int | None = None) -> Dataset:
    """Dataset for a BASELINE.json config; seed = 1000 + config index."""
    c = CONFIGS[name]
    n = c["n_snps"] if n_snps is None else n_snps
    s = 1000 + c["index"] if seed is None else seed
    pq = planted_quad_for(c["n_snps"]) if planted else None
    if pq is not None and pq[-1] >= n:
        pq = None
    return make_dataset(n, c["n_controls"], c["n_cases"], s, planted=pq, uniform=uniform, name=name)


def hand_dataset() -> Dataset:
    """SURVEY.md App. B hand-enumerated dataset (N=4 SNPs, 4 controls + 4 cases).

    Sample order: the 4 controls then the 4 cases as listed there."""
    ctrl = [(0, 0, 0, 0), (0, 0, 0, 0), (1, 2, 0, 1), (2, 2, 2, 2)]
    case = [(0, 0, 0, 0), (1, 2, 0, 1), (1, 2, 0, 1), (0, 1, 2, 0)]
    geno = np.array(ctrl + case, dtype=np.uint8).T.copy()
    phen = np.array([0] * 4 + [1] * 4, dtype=np.uint8)
    return Dataset(geno=geno, phen=phen, n_controls=4, n_cases=4, planted=None, seed=-1, name="hand")
