"""profiles/inst_counts.json from ncu metric CSVs (test/bench infrastructure):
per kernel, warp-level instruction counts per unit of work, for bench.py's
integer-pipe rooflines (alu_roofline).

    python scripts/inst_counts.py <tag> c2=gpurun_out/inst_c2.csv c4=gpurun_out/inst_c4.csv [c4_ncand=N]

Units: c2 -- candidates per launch (the profile_target c2 step: the 64-vector
bench batch, 13^8 candidates each); c4 -- (count vector, demand vector)
evaluations of k_fact_gv (3600 vectors x count vectors per vector)."""
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def read(path):
    rows = {}
    with open(path) as f:
        lines = [ln for ln in f if ln.startswith('"')]
    for r in csv.DictReader(lines):
        k = (r["ID"], r["Kernel Name"])
        rows.setdefault(k, {})[r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
    return rows


def summarise(rows, match, units):
    tot = {}
    n = 0
    for (i, name), m in rows.items():
        if match in name:
            n += 1
            for k, v in m.items():
                tot[k] = tot.get(k, 0.0) + v
    if not n:
        return None
    return {"launches": n, "units_per_launch": units, "alu_per_unit": tot["sm__inst_executed_pipe_alu.sum"] / n / units,
            "fma_per_unit": tot["sm__inst_executed_pipe_fma.sum"] / n / units,
            "inst_per_unit": tot["sm__inst_executed.sum"] / n / units,
            "dram_bytes_per_unit": (tot["dram__bytes_read.sum"] + tot["dram__bytes_write.sum"]) / n / units,
            "local_load_sectors_per_launch": tot.get("l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum", 0) / n,
            "ncu_duration_ns_per_launch": tot["gpu__time_duration.sum"] / n,
            "warps_active_pct": tot.get("sm__warps_active.avg.pct_of_peak_sustained_active", 0) / n}


if __name__ == "__main__":
    tag = sys.argv[1]
    kv = dict(a.split("=", 1) for a in sys.argv[2:])
    out = {}
    if "c2" in kv:
        s = summarise(read(kv["c2"]), "k_flat_", 64 * 13**8)
        if s:
            out["score_flat_pair"] = dict(s, source=f"profiles/{tag}: ncu --metrics on scripts/profile_target.py c2 "
                                                    "(64-vector bench batch), warp instructions / candidates")
    if "c4" in kv:
        units = 3600 * int(kv.get("c4_ncand", 1088010))
        s = summarise(read(kv["c4"]), "k_fact_gv", units)
        if s:
            out["fact_g"] = dict(s, source=f"profiles/{tag}: ncu --metrics on scripts/profile_target.py c4 "
                                           "(3600 vectors), warp instructions / evaluations")
    p = os.path.join(ROOT, "profiles", "inst_counts.json")
    old = json.load(open(p)) if os.path.exists(p) else {}
    old.update(out)
    json.dump(old, open(p, "w"), indent=1)
    print(json.dumps(out, indent=1))
