#!/usr/bin/env python
"""Benchmark of the exhaustive fourth-order K2 search (BASELINE.json metric: tera quads/s scaled to
sample size, C(N,4)*M / t).

  python bench.py --gpus N --steps K --warmup W [--config C5] [--also C2] [--pipe tc] [--impl ours|reference]

A step = one pass of the whole hot path over the config's synthetic dataset:
pack the byte genotypes into bit planes (a1), T1/T2/T3 (a2, a4), the 4-way contraction with the fused
epilogue and top-k (a3, a5-a7), and for N > 1 the all_gather + merge of the per-rank top-k (a8).
`value` is measured with the genotypes already resident in HBM; `e2e` through the same public API from
pinned HOST buffers (H2D of the genotypes and D2H of the result inside the timed region).
For N > 1 (torchrun) the quad space of the same dataset is split across ranks by the static LPT plan:
total work is fixed -> "scaling": "strong" (the paper's Fig. 3 experiment).
`--impl reference` times the CPU oracle (the only reference this tier has) on a bounded sample.

The default workload is C5 (N=1024, M=100003, 30/70): the largest BASELINE.json config one B200 runs within the
driver's step protocol (C3 takes ~165 s per step, C4 is 8-GPU work).  The same run also times C2 (the config
BASELINE.json lists as "single B200") with the same steps / warm-up and reports it under "also" in the same
JSON line (--also none to skip).  `--gpus N` without torchrun relaunches itself under torch.distributed.run.
"""
from __future__ import annotations

import argparse
import gc
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import datagen  # noqa: E402

METRIC = "tera quads/s scaled to sample size (C(N,4)*M/s)"
UNIT = "Tquads/s"


def comb4(n):
    return n * (n - 1) * (n - 2) * (n - 3) // 24


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f), "measured"
    except Exception:
        return {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0,
                "sm_max_mhz": 1965.0}, "fallback"


class ClockSampler:
    """nvidia-smi clocks + throttle reasons sampled every 200 ms while running."""

    def __init__(self, index=0):
        self.index = index
        self.samples = []
        self.proc = None

    def __enter__(self):
        if os.environ.get("EPI4_BENCH_NO_CLOCKS"):   # diagnostics only: no sampler (the line reports "unsampled")
            return self
        q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
             "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
             "clocks_event_reasons.sw_power_cap")
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except Exception:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) >= 7:
                self.samples.append(parts)

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()

    def summary(self):
        if not self.samples:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        sm = [float(s[0]) for s in self.samples if s[0].replace(".", "").isdigit()]
        mx = [float(s[1]) for s in self.samples if s[1].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for s in self.samples for i in range(4) if s[3 + i].lower() == "active"})
        pw = [float(s[2]) for s in self.samples if s[2].replace(".", "").isdigit()]
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "power_w_median": statistics.median(pw) if pw else None,
                "samples": len(self.samples)}


def cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except Exception:
        pass
    return "unknown"


def cpu_oracle_sample(d, target_s=12.0, max_w=None):
    """Time the oracle (as it stands) on the first W SNPs at full M; W picked so it runs ~target_s."""
    import oracle
    cores = oracle.max_threads(0)
    w = 24
    t0 = time.perf_counter()
    oracle.search(d.geno, d.phen, top_k=1, n_snps=w)
    t = time.perf_counter() - t0
    rate = comb4(w) / max(t, 1e-6)
    n = d.n_snps if max_w is None else min(d.n_snps, max_w)
    while w + 1 <= n and comb4(w + 1) / rate < target_s:
        w += 1
    t0 = time.perf_counter()
    oracle.search(d.geno, d.phen, top_k=1, n_snps=w)
    t = time.perf_counter() - t0
    rate = comb4(w) * d.n_samples / t
    full_h = comb4(d.n_snps) * d.n_samples / rate / 3600.0
    return {"value": rate / 1e12, "unit": UNIT, "cores": cores, "kind": "oracle", "cpu_model": cpu_model(),
            "sample": f"exhaustive search over the first {w} SNPs ({comb4(w)} quads) x all M={d.n_samples} "
                      f"samples of {d.name}; {t:.2f} s on {cores} host threads",
            "extrapolated_full_run_hours": full_h}


def flush_l2(torch, buf):
    buf.zero_()   # 512 MiB write > 126 MB L2, outside the timed region


def measure(cfg, args, world, rank, local, torch, dist, epi):
    """W warm-up steps and K timed steps of the whole hot path on config `cfg`; returns the JSON fields."""
    d = datagen.make_config(cfg)
    n, m = d.n_snps, d.n_samples
    stream = torch.cuda.Stream()
    # N > 1: every rank builds the 3-way table on its tensor cores (~3 ms at C2, tiny next to the search);
    # --shard-t3 instead builds 1/world of it per rank (POPC kernel) and all-gathers the shares over NCCL
    shard = world > 1 and args.shard_t3
    eng = epi.Epi4(local, pipe=args.pipe, rank=rank, world=world, shard_t3=shard, objective=args.objective,
                   tile=None if args.tile == "auto" else int(args.tile))
    eng.set_stream(stream.cuda_stream)
    geno_d = torch.from_numpy(d.geno).to(f"cuda:{local}")
    phen_d = torch.from_numpy(d.phen).to(f"cuda:{local}")
    geno_h = torch.from_numpy(d.geno).pin_memory()
    phen_h = torch.from_numpy(d.phen).pin_memory()
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=f"cuda:{local}")
    top_k = args.top_k

    def local_search(k):
        return eng.search(k)

    def step(host):
        if host:
            epi.binding.epi4_pack_genotypes(eng.ctx, geno_h.data_ptr(), phen_h.data_ptr(), n, m,
                                            epi.binding.EPI4_PTR_HOST)
        else:
            eng.load_genotypes(geno_d, phen_d)
        if shard:
            eng.gather_t3()
        if world > 1:
            return epi.search_distributed(local_search, top_k)
        return eng.search(top_k)

    other_ms = []   # per timed step (device steps, then e2e steps): pack + T1/T2/T3 + merge time (library events)

    def timed(host, steps):
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        times, quad_ms, launches, res = [], [], 0, None
        for _ in range(steps):
            flush_l2(torch, flush)
            torch.cuda.synchronize()
            if world > 1:
                dist.barrier()
            ev0.record(stream)
            res = step(host)
            ev1.record(stream)
            torch.cuda.synchronize()
            times.append(ev0.elapsed_time(ev1))
            st = eng.stats()
            quad_ms.append(st["ms_quad"])
            other_ms.append(round(st["ms_pack"] + st["ms_pop"] + st["ms_merge"], 3))
            launches += st["launches"] + st["launches_load"]
        return times, quad_ms, launches, res

    for _ in range(args.warmup):
        step(False)
    torch.cuda.synchronize()
    # Python's cyclic GC is paused over the timed steps (collected just before): a full collection in a process
    # holding torch takes tens of ms and landed inside random steps (profiles/r01i_step_jitter.txt)
    gc.collect()
    gc.disable()
    try:
        with ClockSampler(local) as clk:
            times, quad_ms, launches, res = timed(False, args.steps)
        e2e_times, _, _, _ = timed(True, max(1, min(args.steps, 3)))
    finally:
        gc.enable()
    t_step = statistics.mean(times)
    t_e2e = statistics.mean(e2e_times)
    t_quad = statistics.mean(quad_ms)
    if world > 1:
        tt = torch.tensor([t_step, t_e2e, t_quad], dtype=torch.float64, device=f"cuda:{local}")
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        t_step, t_e2e, t_quad = tt.tolist()
    scaled = comb4(n) * m
    value = scaled / (t_step / 1e3) / 1e12
    e2e = scaled / (t_e2e / 1e3) / 1e12
    st = eng.stats()
    pk, pk_src = peaks()
    useful_macs = 16.0 * comb4(n) * m / world
    if args.pipe == "tc":
        # kind::mxf4 (E2M1 operands): dense fp4 = 4 x bf16 (guide nominal 9 / 2.25 PFLOP/s), sustained
        # figure because the kernel runs for ~1 s or more inside a long step
        peak = 4.0 * pk["bf16_tflops_sustained"]
        bound, unit = "tensor", "TFLOP/s"
        achieved = 2.0 * useful_macs / (t_quad / 1e3) / 1e12  # fp4 ops (2 per {0,1}-MAC) per second
        peak_note = f"{pk_src} bf16_tflops_sustained x 4 (fp4/bf16 nominal ratio, kind::mxf4)"
    else:
        # ALU-bound popcount pipe: 16 POPC/clk/SM x 32 bit-MACs x 148 SMs x sm_max clock, 2 ops per MAC
        peak = 2.0 * 16 * 32 * 148 * pk.get("sm_max_mhz", 1965.0) * 1e6 / 1e12
        bound, unit = "alu", "TFLOP/s"
        achieved = 2.0 * useful_macs / (t_quad / 1e3) / 1e12
        peak_note = "derived: 16 POPC/clk/SM x 32 x 148 SMs x sm_max_mhz, 2 ops per bit-MAC"
    traffic = None
    tf = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tf):
        try:
            traffic = json.load(open(tf)).get(f"{cfg}:{args.pipe}")
        except Exception:
            traffic = None
    out = {
        "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": t_step, "higher_is_better": True, "scaling": "strong",
        "vs_baseline": None, "dtype": "e2m1 (mxf4, f32 accum)" if args.pipe == "tc" else "u32",
        "data": "synthetic (seeded HWE genotypes + planted 4-way interaction, SURVEY.md §8(d))",
        "config": {"workload": f"{cfg}: N={n} SNPs, M={m} samples ({d.n_controls} controls / "
                               f"{d.n_cases} cases), exhaustive C(N,4)={comb4(n)} quads, top_k={top_k}",
                   "pipe": args.pipe, "objective": args.objective,
                   "tile_n": int(st.get("tile_n", 0)),
                   "parallelism": f"static LPT over (w-block, x) units x {world} ranks (NCCL world {world})" +
                                  (", T3 sharded + NCCL all_gather" if shard else ""),
                   "l2": "flushed (512 MiB write) before every timed step"},
        "e2e": {"value": e2e, "unit": UNIT, "h2d_bytes_per_step": int(n * m + m),
                "d2h_bytes_per_step": int(top_k * 16 + 4)},
        "gpu_launches": int(launches),
        "roofline": {"bound": bound, "achieved": achieved, "peak": peak, "unit": unit,
                     "frac": achieved / peak, "traffic": traffic,
                     "kernel": f"k_quad_{args.pipe}", "kernel_ms": t_quad,
                     "algorithmic": "16 {0,1}-MACs per (quad, sample): 16*C(N,4)*M/world per launch",
                     "peak_source": peak_note},
        "breakdown_ms": {"pack": st["ms_pack"], "pop_T1T2T3": st["ms_pop"], "quad": st["ms_quad"],
                         "merge_d2h": st["ms_merge"]},
        "step_ms": [round(t, 3) for t in times], "e2e_step_ms": [round(t, 3) for t in e2e_times],
        "quad_step_ms": [round(t, 3) for t in quad_ms], "load_merge_step_ms": other_ms,
        "useful_over_executed": (16.0 * st["quads"] * (d.n_controls + d.n_cases)) / max(st["executed_macs"], 1.0),
        "clocks": clk.summary(),
        "best": {"quad": epi.unpack_index(res[0][0]), "key": float(res[1][0])}
        if args.objective != "k2" else {"quad": epi.unpack_index(res[0][0]), "k2": float(res[1][0])},
    }
    if args.pipe == "tc":
        # second denominator: the microbenchmarked MMA rate at the clock logged during the timed region —
        # kind::mxf4 M=256 K=64 issues in N/2 cycles per SM pair (tools/probe_mxf4b.cu), i.e. 128 x 64 x 2 MACs
        # per SM and cycle whatever N = 2 x 16384 fp4 ops per SM and cycle
        mhz = out["clocks"].get("sm_mhz") or pk.get("sm_max_mhz", 1965.0)
        probe = 2.0 * 16384 * 148 * float(mhz) * 1e6 / 1e12
        out["roofline"]["peak_probe"] = probe
        out["roofline"]["frac_probe"] = achieved / probe
        out["roofline"]["peak_probe_source"] = (f"tools/probe_mxf4b.cu MMA rate (16384 {{0,1}}-MACs/clk/SM) x 148 SMs x "
                                                f"{mhz:.0f} MHz median SM clock of the timed region")
    if rank == 0 and world == 1 and not args.no_cpu_baseline:
        out["cpu_baseline"] = cpu_oracle_sample(d)
    eng.close()
    del geno_d, phen_d, flush
    torch.cuda.empty_cache()
    return out


def run_ours(args):
    import torch
    import torch.distributed as dist
    import paper_conf_icpp_nobreiss22_b200 as epi

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    if world != args.gpus:
        print(f"bench.py: --gpus {args.gpus} but WORLD_SIZE={world}", file=sys.stderr)
        sys.exit(2)
    torch.cuda.set_device(local)
    if world > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        assert dist.get_world_size() == world
    out = measure(args.config, args, world, rank, local, torch, dist, epi)
    if args.also not in ("none", "", args.config):
        sec = measure(args.also, args, world, rank, local, torch, dist, epi)
        out["also"] = {k: sec[k] for k in ("config", "value", "unit", "ms_per_step", "e2e", "roofline", "step_ms",
                                           "quad_step_ms", "useful_over_executed", "clocks", "best",
                                           "breakdown_ms", "gpu_launches") if k in sec}
        if "cpu_baseline" in sec:
            out["also"]["cpu_baseline"] = sec["cpu_baseline"]
    if rank == 0:
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


def relaunch(args):
    """`--gpus N` without torchrun: run N ranks under torch.distributed.run on this node (127.0.0.1)."""
    import socket
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
           "--master-addr", "127.0.0.1", "--master-port", str(port), os.path.abspath(__file__)] + sys.argv[1:]
    sys.exit(subprocess.call(cmd))


def run_reference(args):
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    d = datagen.make_config(args.config)
    cores = oracle.max_threads(0)
    # size one step so the whole run stays within a few minutes
    nsteps = args.warmup + args.steps
    probe = cpu_oracle_sample(d, target_s=max(2.0, min(20.0, 150.0 / max(nsteps, 1))))
    w = int(probe["sample"].split("first ")[1].split(" SNPs")[0])
    for _ in range(args.warmup):
        oracle.search(d.geno, d.phen, top_k=1, n_snps=w)
    ts = []
    for _ in range(args.steps):
        t0 = time.perf_counter()
        oracle.search(d.geno, d.phen, top_k=1, n_snps=w)
        ts.append(time.perf_counter() - t0)
    t = statistics.mean(ts)
    value = comb4(w) * d.n_samples / t / 1e12
    sample = f"exhaustive oracle search over the first {w} SNPs ({comb4(w)} quads) x all M={d.n_samples} samples"
    print(json.dumps({
        "impl": "reference", "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world,
        "steps": args.steps, "warmup": args.warmup, "ms_per_step": t * 1e3, "higher_is_better": True,
        "scaling": "strong", "vs_baseline": None, "dtype": "u8", "data": "synthetic",
        "config": {"workload": f"{args.config}: N={d.n_snps}, M={d.n_samples}; CPU oracle on a bounded sample"},
        "cpu_baseline": {"value": value, "unit": UNIT, "cores": cores, "kind": "oracle", "sample": sample,
                         "cpu_model": cpu_model(),
                         "extrapolated_full_run_hours": comb4(d.n_snps) * d.n_samples / (value * 1e12) / 3600.0},
        "e2e": {"value": value, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
    }), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C5", choices=list(datagen.CONFIGS))
    ap.add_argument("--also", default="C2", help="second config timed in the same run, reported under 'also' "
                    "(none to skip)")
    ap.add_argument("--pipe", default="tc", choices=["tc", "lop3"])
    ap.add_argument("--top-k", type=int, default=16)
    ap.add_argument("--tile", default="auto", choices=["auto", "128", "224"],
                    help="tensor-core tile geometry (default: chosen by the load from the sample counts)")
    ap.add_argument("--objective", default="k2", choices=["k2", "mi", "chi2"],
                    help="ranking objective (K2 is the paper's and the headline; MI / chi-square: SURVEY §8(f) NEXT-4)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--shard-t3", action="store_true", help="N > 1: build 1/world of the 3-way table per rank and "
                    "all-gather the shares (NCCL) instead of building it on every rank")
    args = ap.parse_args()
    if args.warmup < 3 and args.impl == "ours":
        print("warning: --warmup < 3 violates the timing rules", file=sys.stderr)
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        relaunch(args)
    (run_reference if args.impl == "reference" else run_ours)(args)


if __name__ == "__main__":
    main()
