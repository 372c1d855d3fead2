"""Single-search measurements beside the bench line: the larger BASELINE configs (C3, C5) and
the C5 sample-count sweep (N = 1024, 30/70 cases/controls, M in {16384 .. 100003}).

  python tools/sweep.py [--what sweep,C3,C5] [--out gpurun_out/sweep.jsonl]

Each point: one untimed warm-up search on C1, then load + one full search of the point's dataset; the
search's own CUDA-event timing of the contraction kernel (stats ms_quad) and the wall time of the whole
search call are reported as scaled quads/s, C(N,4)*M / t, with the kernel's fraction of the fp4 tensor peak
(16 {0,1}-MACs per quad and sample, 2 ops per MAC, against 4 x MEASURED_PEAKS bf16_tflops_sustained, as in
bench.py).  These are single measurements, not bench lines (no warm-up steps / L2 flush protocol).
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


def peak_tflops():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return 4.0 * json.load(f)["bf16_tflops_sustained"], "measured bf16_tflops_sustained x 4"
    except Exception:
        return 4.0 * 1400.0, "fallback 1400 x 4"


def point(name, d, top_k=16):
    n, m = d.n_snps, d.n_samples
    with epi.Epi4(0, pipe="tc") as e:
        e.load_genotypes(d.geno, d.phen)
        t0 = time.perf_counter()
        idx, k2 = e.search(top_k)
        wall = time.perf_counter() - t0
        st = e.stats()
    q = math.comb(n, 4) * m
    kern_s = st["ms_quad"] / 1e3
    peak, src = peak_tflops()
    ach = 2.0 * 16.0 * q / kern_s / 1e12
    best = epi.unpack_index(idx[0]) if len(idx) else None
    return {"point": name, "n_snps": n, "m": m, "n_controls": d.n_controls, "n_cases": d.n_cases,
            "tquads_per_s_kernel": q / kern_s / 1e12, "tquads_per_s_search": q / wall / 1e12,
            "kernel_ms": st["ms_quad"], "search_wall_s": wall, "roofline_frac": ach / peak,
            "achieved_tflops": ach, "peak_tflops": peak, "peak_source": src,
            "useful_over_executed": st["quads"] * 16.0 * m / st["executed_macs"] if st["executed_macs"] else None,
            "best": {"quad": best, "k2": float(k2[0]) if len(k2) else None}, "planted": d.planted}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--what", default="sweep,C5,C3")
    ap.add_argument("--out", default=os.path.join(ROOT, "gpurun_out", "sweep.jsonl"))
    a = ap.parse_args()
    os.makedirs(os.path.dirname(a.out), exist_ok=True)
    with epi.Epi4(0, pipe="tc") as e:   # warm-up (module load, first-launch costs)
        c1 = datagen.make_config("C1")
        e.load_genotypes(c1.geno, c1.phen)
        e.search(4)
    todo = []
    for w in a.what.split(","):
        if w == "sweep":
            for m in (16384, 32768, 65536, 100003):
                n1 = int(round(0.3 * m))
                todo.append((f"C5-sweep M={m}", lambda m=m, n1=n1: datagen.make_dataset(
                    1024, m - n1, n1, 2000 + m, planted=datagen.planted_quad_for(1024), name=f"sweep{m}")))
        elif w == "paper2048":
            # the paper's single-GPU shape (2048 SNPs, balanced; P:L264-266 used M = 524288) at the largest M the
            # packed 32-bit counts allow (65535 per class)
            todo.append(("paper-shape N=2048 M=131070", lambda: datagen.make_dataset(
                2048, 65535, 65535, 3000, planted=datagen.planted_quad_for(2048), name="paper2048")))
        else:
            todo.append((w, lambda w=w: datagen.make_config(w)))
    with open(a.out, "a") as f:
        for name, mk in todo:
            r = point(name, mk())
            print(json.dumps(r), flush=True)
            f.write(json.dumps(r) + "\n")


if __name__ == "__main__":
    main()
