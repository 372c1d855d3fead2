"""Merge per-rank full_search records (tools/full_search.py --rank r --world W, run one after the other on one GPU)
into the record of the whole search: the exact global top-16 by (K2, index) (merge_topk, the merge of the
multi-GPU path), the planted-quad check, and the throughput of the whole search on one GPU (all quads x M over
the sum of the ranks' kernel times) and, as W GPUs would run it, over the slowest rank's kernel time.

  python tools/merge_ranks.py profiles/r02l_full_C4.jsonl
"""
import json
import sys

import numpy as np

sys.path.insert(0, __import__("os").path.dirname(__import__("os").path.dirname(__import__("os").path.abspath(__file__))))
import paper_conf_icpp_nobreiss22_b200 as epi  # noqa: E402

recs = [json.loads(l) for l in open(sys.argv[1]) if l.strip()]
recs = [r for r in recs if r.get("world", 1) > 1]
world = recs[0]["world"]
assert sorted(r["rank"] for r in recs) == list(range(world)), "need every rank once"
parts = [(np.array(r["top16_packed"], dtype=np.uint64), np.array([k for _, k in r["top16"]])) for r in recs]
idx, k2 = epi.merge_topk(parts, 16)
quads = sum(r["quads"] for r in recs)
m = recs[0]["m"]
ksum = sum(r["kernel_ms"] for r in recs) / 1e3
kmax = max(r["kernel_ms"] for r in recs) / 1e3
best = epi.unpack_index(int(idx[0]))
out = {"point": recs[0]["point"].split(" rank")[0] + f" (all {world} ranks, merged)", "n_snps": recs[0]["n_snps"],
       "m": m, "quads": quads, "full_quads": recs[0]["full_quads"], "complete": quads == recs[0]["full_quads"],
       "tquads_per_s_one_gpu": quads * m / ksum / 1e12, "kernel_s_sum": ksum,
       "tquads_per_s_if_parallel": quads * m / kmax / 1e12, "kernel_s_max": kmax,
       "rank_balance_max_over_mean": kmax / (ksum / world),
       "best": {"quad": best, "k2": float(k2[0])}, "planted": recs[0]["planted"],
       "planted_is_argmin": recs[0]["planted"] is not None and list(best) == list(recs[0]["planted"]),
       "top16": [[epi.unpack_index(int(i)), float(k)] for i, k in zip(idx, k2)],
       "clocks": [r["clocks"] for r in recs], "sources": [r.get("source") for r in recs]}
print(json.dumps(out))
