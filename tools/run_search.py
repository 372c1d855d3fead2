"""One search on a config (optionally a slice of the plan's units) — the command ncu wraps."""
import argparse
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import datagen  # noqa: E402
import paper_conf_icpp_nobreiss22_b200 as epi  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C2")
ap.add_argument("--pipe", default="tc")
ap.add_argument("--units", type=int, default=-1, help="first U units of the plan (-1 = all)")
ap.add_argument("--top-k", type=int, default=16)
ap.add_argument("--repeat", type=int, default=1)
ap.add_argument("--debug", type=int, default=0)
ap.add_argument("--grid", type=int, default=0)
ap.add_argument("--objective", default="k2", choices=["k2", "mi", "chi2"])
ap.add_argument("--tile", type=int, default=None, help="force the tensor-core tile geometry (128 / 224)")
ap.add_argument("--n-snps", type=int, default=None, help="first N SNPs of the config's dataset (all M samples)")
a = ap.parse_args()
d = datagen.make_config(a.config, n_snps=a.n_snps)
with epi.Epi4(0, pipe=a.pipe, debug=a.debug, grid=a.grid, objective=a.objective, tile=a.tile) as e:
    e.load_genotypes(d.geno, d.phen)
    for _ in range(a.repeat):
        t0 = time.time()
        idx, k2 = e.search_units(0, a.units, a.top_k) if a.units >= 0 else e.search(a.top_k)
        st = e.stats()
        best = (epi.unpack_index(idx[0]), float(k2[0])) if len(idx) else None
        print(f"{a.config} {a.pipe} {a.objective} dbg={a.debug}: best {best} quad {st['ms_quad']:.2f} ms "
              f"N {st['tile_n']} tiles {st['tiles']} quads {st['quads']} wall {time.time() - t0:.2f}s prof {[f'{v:.3g}' for v in st['prof']]}", flush=True)
