"""Summarise ncu captures (run here, on the CPU box) into profiles/.

    python scripts/ncu_summary.py <round tag> gpurun_out/full_*.ncu-rep gpurun_out/launches_*.csv

Writes profiles/<tag>_kernels.json / .md (per-kernel counters from the full
captures) and profiles/<tag>_launches.md (per-kernel share of each launch
list; ncu launch times are cold-cache and serialised: compare shares).
"""

import collections
import csv
import io
import json
import os
import subprocess
import sys

METRICS = {
    "duration_us": ("gpu__time_duration.sum", 1e-3),
    "ipc_per_sm": ("sm__inst_executed.avg.per_cycle_active", 1),
    "issue_active_pct": ("smsp__issue_active.avg.pct_of_peak_sustained_active", 1),
    "warps_active_per_sm": ("sm__warps_active.avg.per_cycle_active", 1),
    "alu_pipe_pct": ("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", 1),
    "fma_pipe_pct": ("sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", 1),
    "sm_throughput_pct": ("sm__throughput.avg.pct_of_peak_sustained_elapsed", 1),
    "dram_read_bytes": ("dram__bytes_read.sum", 1),
    "dram_write_bytes": ("dram__bytes_write.sum", 1),
    "dram_throughput_pct": ("dram__throughput.avg.pct_of_peak_sustained_elapsed", 1),
    "registers": ("launch__registers_per_thread", 1),
    "block": ("launch__block_size", 1),
    "grid": ("launch__grid_size", 1),
    "warp_instructions": ("smsp__inst_executed.sum", 1),
    "local_load_sectors": ("l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum", 1),
    "smem_bank_conflicts": ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", 1),
}
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1, "us": 1e3, "ms": 1e6, "s": 1e9,
        "nsecond": 1, "usecond": 1e3, "msecond": 1e6}


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        k = {"kernel": r[hdr.index("Kernel Name")][:60]}
        for name, (m, scale) in METRICS.items():
            if m in hdr:
                i = hdr.index(m)
                try:
                    v = float(r[i].replace(",", ""))
                except ValueError:
                    continue
                if units[i] in UNIT and name.endswith(("bytes", "_us")):
                    v *= UNIT[units[i]]
                k[name] = v * scale if name != "duration_us" else v / 1e3
        stalls = {}  # warp-cycles stalled per issued instruction, by reason
        for i, h in enumerate(hdr):
            if h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio"):
                reason = h[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]
                if reason in ("selected",):
                    continue
                try:
                    stalls[reason] = float(r[i])
                except ValueError:
                    pass
        k["top_stalls_pct"] = dict(sorted(stalls.items(), key=lambda x: -x[1])[:5])
        res.append(k)
    return res


def launches(path):
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    hdr = rows[0]
    ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    agg = collections.OrderedDict()
    for r in rows[1:]:
        name = r[ki].split("(")[0][:48]
        v = float(r[vi].replace(",", "")) * UNIT.get(r[ui], 1) / 1e3  # us
        agg.setdefault(name, []).append(v)
    tot = sum(sum(v) for v in agg.values())
    return [(k, len(v), sum(v) / len(v), sum(v), 100 * sum(v) / tot) for k, v in agg.items()], tot


def main():
    tag = sys.argv[1]
    os.makedirs("profiles", exist_ok=True)
    kern, md = [], [f"# ncu per-kernel counters ({tag})\n", "Full captures (`ncu --set full --clock-control none`,"
                    " one launch each, replayed; times are cold-cache and serialised).\n",
                    "| kernel | us | IPC/SM | issue % | warps/SM | ALU % | FMA % | DRAM R+W GB | regs | top stalls (cycles per issue) |",
                    "|---|---|---|---|---|---|---|---|---|---|"]
    lmd = [f"# ncu launch lists ({tag})\n", "`ncu --metrics gpu__time_duration.sum --clock-control none`: per-launch "
           "times are cold-cache and serialised -- compare the shares, not the absolutes.\n"]
    for p in sys.argv[2:]:
        if p.endswith(".ncu-rep"):
            for k in raw(p):
                k["source"] = os.path.basename(p)
                kern.append(k)
                g = lambda n, f="{:.1f}": f.format(k[n]) if n in k else "-"
                dr = (k.get("dram_read_bytes", 0) + k.get("dram_write_bytes", 0)) / 1e9
                st = ", ".join(f"{a} {b:.2f}" for a, b in list(k["top_stalls_pct"].items())[:3])
                md.append(f"| {k['kernel'][:40]} | {g('duration_us')} | {g('ipc_per_sm', '{:.2f}')} | "
                          f"{g('issue_active_pct')} | {g('warps_active_per_sm')} | {g('alu_pipe_pct')} | "
                          f"{g('fma_pipe_pct')} | {dr:.3f} | {g('registers', '{:.0f}')} | {st} |")
        elif p.endswith(".csv"):
            rows, tot = launches(p)
            lmd += [f"## {os.path.basename(p)} (total {tot:.1f} us)\n", "| kernel | launches | mean us | total us | share % |",
                    "|---|---|---|---|---|"]
            lmd += [f"| {k} | {n} | {m:.1f} | {t:.1f} | {s:.1f} |" for k, n, m, t, s in rows]
            lmd.append("")
    json.dump(kern, open(f"profiles/{tag}_kernels.json", "w"), indent=1)
    open(f"profiles/{tag}_kernels.md", "w").write("\n".join(md) + "\n")
    open(f"profiles/{tag}_launches.md", "w").write("\n".join(lmd) + "\n")
    print("\n".join(md))
    print("\n".join(lmd))


if __name__ == "__main__":
    main()
