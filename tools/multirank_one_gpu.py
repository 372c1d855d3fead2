"""Exercise the N > 1 path of bench.py: torchrun --nproc-per-node W.  Each rank builds its share of T3, the
shares are all-gathered (Epi4.gather_t3), every rank searches its LPT units, and the per-rank top-k lists are
all-gathered and merged (search_distributed).  Rank 0 compares the result with a 1-rank search.
  --backend gloo (default): every rank on cuda:0 (NCCL refuses two ranks on one device), collectives staged
                            through the host;
  --backend nccl          : rank r on cuda:LOCAL_RANK, device-tensor collectives over NVLink (needs W GPUs).

  torchrun --standalone --nproc-per-node 2 tools/multirank_one_gpu.py [--backend nccl] [--config C2] [--n-snps 160]
"""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402
import torch  # noqa: E402
import torch.distributed as dist  # noqa: E402

import datagen  # noqa: E402
import paper_conf_icpp_nobreiss22_b200 as epi  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--n-snps", type=int, default=160)
ap.add_argument("--top-k", type=int, default=16)
ap.add_argument("--backend", default="gloo", choices=["gloo", "nccl"])
a = ap.parse_args()
dev = int(os.environ.get("LOCAL_RANK", "0")) if a.backend == "nccl" else 0
torch.cuda.set_device(dev)
dist.init_process_group(a.backend)
rank, world = dist.get_rank(), dist.get_world_size()
d = datagen.make_config(a.config, n_snps=a.n_snps)
with epi.Epi4(dev, pipe="tc", rank=rank, world=world, shard_t3=True) as e:
    e.load_genotypes(d.geno, d.phen)
    e.gather_t3()
    idx, k2 = epi.search_distributed(e.search, a.top_k, device="cuda" if a.backend == "nccl" else "cpu")
if rank == 0:
    with epi.Epi4(dev, pipe="tc") as e1:
        e1.load_genotypes(d.geno, d.phen)
        ridx, rk2 = e1.search(a.top_k)
    ok = np.array_equal(idx, ridx) and np.array_equal(k2, rk2)
    print(f"multirank {a.backend} world={world} {a.config} N={d.n_snps}: {'OK' if ok else 'MISMATCH'} "
          f"best {epi.unpack_index(idx[0])} {k2[0]:.6f}", flush=True)
    if not ok:
        sys.exit(1)
dist.destroy_process_group()
