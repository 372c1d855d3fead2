"""Full C4 exhaustive search (N = 4096, M = 65536: C(4096,4) = 1.17e13 quads) on ONE B200 with the windowed
3-way table, in plan chunks (search_units) whose per-chunk results are appended to the output as they
finish; the last line merges them (top-k by (K2, index)).  C4 is an 8-GPU config in BASELINE.json; this run
shows the single-GPU path end to end.

  python tools/c4_full.py [--chunks 4] [--out gpurun_out/c4_full.jsonl]
"""
import argparse
import json
import math
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import datagen  # noqa: E402
import paper_conf_icpp_nobreiss22_b200 as epi  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--chunks", type=int, default=4)
ap.add_argument("--begin", type=int, default=0, help="first plan unit (a later call resumes)")
ap.add_argument("--end", type=int, default=-1)
ap.add_argument("--top-k", type=int, default=16)
ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "c4_full.jsonl"))
a = ap.parse_args()
os.makedirs(os.path.dirname(a.out), exist_ok=True)
d = datagen.make_config("C4")
n, m = d.n_snps, d.n_samples
nunits = epi.binding.epi4_plan_count(n)
end = nunits if a.end < 0 else a.end
bounds = [a.begin + round(i * (end - a.begin) / a.chunks) for i in range(a.chunks + 1)]
parts, tot_ms, tot_q, wall0 = [], 0.0, 0, time.time()
with epi.Epi4(0, pipe="tc") as e:
    t0 = time.time()
    e.load_genotypes(d.geno, d.phen)
    load_s = time.time() - t0
    for c in range(a.chunks):
        t0 = time.time()
        idx, k2 = e.search_units(bounds[c], bounds[c + 1], a.top_k)
        st = e.stats()
        parts.append((idx, k2))
        tot_ms += st["ms_quad"]
        tot_q += st["quads"]
        r = {"chunk": c, "units": [bounds[c], bounds[c + 1]], "quads": st["quads"], "kernel_ms": st["ms_quad"],
             "wall_s": time.time() - t0, "best": [epi.unpack_index(idx[0]), float(k2[0])] if len(idx) else None}
        print(json.dumps(r), flush=True)
        with open(a.out, "a") as f:
            f.write(json.dumps(r) + "\n")
# merge every chunk record in the output file (chunks of earlier calls included)
recs = [json.loads(l) for l in open(a.out) if l.strip() and '"chunk"' in l]
covered = sorted(tuple(r["units"]) for r in recs)
idx, k2 = epi.merge_topk(parts, a.top_k)
tot_ms = sum(r["kernel_ms"] for r in recs)
tot_q = sum(r["quads"] for r in recs)
best = min(((r["best"][1], epi.pack_index(*r["best"][0])) for r in recs if r["best"]), default=None)
full = math.comb(n, 4)
r = {"workload": f"C4 full: N={n}, M={m} ({d.n_controls}/{d.n_cases}), all C(N,4) quads on one B200, windowed T3",
     "chunks": covered, "quads": tot_q, "all_quads_covered": tot_q == full, "kernel_s": tot_ms / 1e3,
     "tquads_per_s": tot_q * m / (tot_ms / 1e3) / 1e12 if tot_ms else None,
     "best": [epi.unpack_index(best[1]), best[0]] if best else None, "planted": d.planted, "load_s": load_s}
print(json.dumps(r), flush=True)
with open(a.out, "a") as f:
    f.write(json.dumps(r) + "\n")
