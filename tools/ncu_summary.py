"""Summaries kept under profiles/ (read here from gpurun_out/):

  python tools/ncu_summary.py launches <launches.csv> <title>       -> per-kernel share of the launch list
  python tools/ncu_summary.py full <report.ncu-rep> <title>          -> key metrics of a --set full capture
  python tools/ncu_summary.py stalls <report.ncu-rep>                -> stall samples per barrier wait site

The launch list comes from `ncu --metrics gpu__time_duration.sum --clock-control none` (cold-cache,
serialised launches: compare SHARES of the step, not absolute times).
"""
import csv
import io
import subprocess
import sys
from collections import defaultdict

KEYS = [
    "gpu__time_duration.sum",
    "sm__cycles_elapsed.avg.per_second",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
    "l1tex__m_xbar2l1tex_read_bytes.sum.per_second",
    "l1tex__m_xbar2l1tex_read_bytes_mem_global_op_tma_ld.sum.per_second",
    "l1tex__t_sector_pipe_lsu_mem_global_op_ld_hit_rate.pct",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed",
    "lts__t_sector_hit_rate.pct",
    "dram__bytes_read.sum",
    "dram__bytes_write.sum",
    "smsp__sass_inst_executed_op_local_ld.sum",
    "smsp__sass_inst_executed_op_local_st.sum",
    "launch__registers_per_thread",
    "launch__grid_size",
    "launch__block_size",
]


def ncu_csv(rep, *args):
    out = subprocess.run(["ncu", "-i", rep, *args, "--csv"], capture_output=True, text=True, check=True).stdout
    return list(csv.reader(io.StringIO(out)))


def launches(path, title):
    rows = list(csv.reader(open(path)))
    hdr_i = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[hdr_i]
    k, mn, mv = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    tot, cnt = defaultdict(float), defaultdict(int)
    for r in rows[hdr_i + 1:]:
        if len(r) == len(hdr) and r[mn] == "gpu__time_duration.sum":
            v = float(r[mv].replace(",", ""))
            tot[r[k]] += v
            cnt[r[k]] += 1
    s = sum(tot.values())
    print(f"# {title}")
    print("# gpu__time_duration.sum, --clock-control none; cold-cache serialised launches: compare SHARES, not absolutes")
    print("kernel | launches | total ns | share")
    for name, v in sorted(tot.items(), key=lambda kv: -kv[1]):
        print(f"{name[:90]} | {cnt[name]} | {v:.0f} | {100 * v / s:.2f}%")


def full(rep, title):
    rows = ncu_csv(rep, "--page", "raw")
    hdr, units, vals = rows[0], rows[1], rows[2]
    d = {h: (u, v) for h, u, v in zip(hdr, units, vals)}
    print(f"# {title}")
    for key in KEYS:
        if key in d:
            print(f"{key} [{d[key][0]}] = {d[key][1]}")


def stalls(rep):
    rows = ncu_csv(rep, "--page", "source", "--print-source", "sass")
    hdr = rows[1]
    data = [r for r in rows[2:] if len(r) == len(hdr)]
    i_s, i_src, i_e = hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Source"), hdr.index("Instructions Executed")
    tot = sum(float(r[i_s] or 0) for r in data)
    print(f"total stall samples {tot:.0f}")
    k = 0
    while k < len(data):
        s = data[k][i_src]
        if "TRYWAIT" in s and "TRYWAIT" not in data[k - 1][i_src]:
            j, acc = k, 0.0
            while j < len(data) and j < k + 40 and "BPT.TRAP" not in data[j][i_src]:
                acc += float(data[j][i_s] or 0)
                j += 1
            print(f"wait site sass#{k}: {100 * acc / tot:5.1f}% of samples, executed {data[k][i_e]}")
            k = j
        k += 1
    cls, ex = defaultdict(float), defaultdict(float)
    for r in data:
        op = r[i_src].strip().split()[0] if r[i_src].strip() else "?"
        if op.startswith("@"):
            op = r[i_src].strip().split()[1]
        op = op.split(".")[0]
        cls[op] += float(r[i_s] or 0)
        ex[op] += float(r[i_e] or 0)
    print("by opcode (stall %, executed warp-instr):")
    for op, v in sorted(cls.items(), key=lambda kv: -kv[1])[:20]:
        print(f"  {op:10s} {100 * v / tot:5.1f}%  {ex[op]:.3g}")


if __name__ == "__main__":
    mode = sys.argv[1]
    if mode == "launches":
        launches(sys.argv[2], sys.argv[3])
    elif mode == "full":
        full(sys.argv[2], sys.argv[3])
    else:
        stalls(sys.argv[2])
