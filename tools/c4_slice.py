"""C4 (N = 4096 SNPs, M = 65536 samples) on ONE B200: the resident 3-way table would need 367 GB, so the load
switches to the windowed table (two 34 GB slabs rebuilt on the tensor cores).  A full C4
search is 8-GPU work (~11 min there, ~90 min here), so this searches a contiguous slice of the 1-rank plan
and reports the slice's throughput in the bench unit (useful quads x M / time), slab rebuilds included.

  python tools/c4_slice.py [--begin 6000] [--units 200] [--out gpurun_out/c4_slice.jsonl]
"""
import argparse
import json
import math
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import datagen  # noqa: E402
import paper_conf_icpp_nobreiss22_b200 as epi  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--begin", type=int, default=6000)
ap.add_argument("--units", type=int, default=200)
ap.add_argument("--top-k", type=int, default=16)
ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "c4_slice.jsonl"))
a = ap.parse_args()
t0 = time.time()
d = datagen.make_config("C4")
t_gen = time.time() - t0
nunits = epi.binding.epi4_plan_count(d.n_snps)
with epi.Epi4(0, pipe="tc") as e:
    t0 = time.time()
    e.load_genotypes(d.geno, d.phen)
    t_load = time.time() - t0
    t0 = time.time()
    idx, k2 = e.search_units(a.begin, a.begin + a.units, a.top_k)
    wall = time.time() - t0
    st = e.stats()
m = d.n_samples
r = {"workload": f"C4 slice: plan units [{a.begin}, {a.begin + a.units}) of {nunits}, N={d.n_snps}, M={m}",
     "quads": st["quads"], "tiles": st["tiles"], "search_wall_s": wall, "kernel_ms": st["ms_quad"],
     "tquads_per_s": st["quads"] * m / (st["ms_quad"] / 1e3) / 1e12,
     "tquads_per_s_wall": st["quads"] * m / wall / 1e12,
     "note": "kernel_ms spans the slab rebuilds (3-way-table mode launches) and the search launches",
     "load_s": t_load, "gen_s": t_gen, "launches": st["launches"],
     "best": {"quad": epi.unpack_index(idx[0]) if len(idx) else None, "k2": float(k2[0]) if len(k2) else None},
     "full_c4_quads": math.comb(d.n_snps, 4)}
print(json.dumps(r), flush=True)
os.makedirs(os.path.dirname(a.out), exist_ok=True)
with open(a.out, "a") as f:
    f.write(json.dumps(r) + "\n")
