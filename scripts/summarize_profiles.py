"""Summarise a round's GPU evidence into profiles/ (committed).

    python scripts/summarize_profiles.py <round-tag>

Reads gpurun_out/{bench.json, bench.err, launches.csv, prof_top.ncu-rep} and writes
profiles/<tag>_bench.json, profiles/<tag>_launches.md, profiles/<tag>_ncu_top.md and
profiles/traffic.json (DRAM bytes per launch of the top kernels, read by bench.py).
"""
import csv
import io
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
CONFIG_KEY = "c4-terabyte-r64"                 # the workload round_profile.sh captures
PROF = os.path.join(ROOT, "profiles")
STAGE_OF = {"k_tc_bwd2": "bwd_prefix", "k_tc_p": "fwd_prefix", "k_rows_bwd": "bwd_rows",
            "k_rows_fwd": "fwd_rows", "k_group_bwd": "bwd_prefix", "k_group_fwd": "fwd_prefix",
            "k_prefix_bwd": "bwd_prefix", "k_prefix_fwd": "fwd_prefix", "k_rows_fwd2": "fwd_rows",
            "k_rows_bwd2": "bwd_rows", "k_agg_scatter": "agg", "k_pool": "pool",
            "k_build_keys": "build_keys"}


def short(name):
    n = name.split("(")[0]
    n = n.replace("void ", "").replace("ttemb::", "").replace("<unnamed>::", "")
    return n.strip()[:48]


def launches(tag):
    path = os.path.join(OUT, "launches.csv")
    if not os.path.exists(path):
        return
    rows = list(csv.reader(open(path)))
    h = None
    agg, order = {}, []
    for r in rows:
        if "Kernel Name" in r:
            h = r
            continue
        if h and len(r) == len(h):
            n = short(r[h.index("Kernel Name")])
            if n.startswith("at::"):      # bench.py's untimed L2 flush (torch fill), not our kernels
                continue
            v = float(r[h.index("Metric Value")].replace(",", ""))
            if n not in agg:
                agg[n] = [0.0, 0]
                order.append(n)
            agg[n][0] += v
            agg[n][1] += 1
    tot = sum(v[0] for v in agg.values())
    lines = [f"# {tag}: ncu launch list (gpu__time_duration.sum, --clock-control none)", "",
             "Cold-cache, serialised replay of one bench step (c4); compare shares, not absolutes.",
             "The bench's untimed L2-flush fill (at::FillFunctor) is excluded.", "",
             "| kernel | launches | us / launch | share |", "|---|---|---|---|"]
    for n in sorted(order, key=lambda k: -agg[k][0]):
        v, c = agg[n]
        lines.append(f"| `{n}` | {c} | {v / c / 1e3:.1f} | {100 * v / tot:.1f} % |")
    lines.append(f"| **total** | {sum(v[1] for v in agg.values())} | {tot / 1e3:.1f} | 100 % |")
    open(os.path.join(PROF, f"{tag}_launches.md"), "w").write("\n".join(lines) + "\n")


def ncu_rows():
    """Rows of every prof_top*.ncu-rep (first launch of each kernel name wins)."""
    h = units = None
    out, seen = [], set()
    for f in sorted(os.listdir(OUT)):
        if not (f.startswith("prof_top") and f.endswith(".ncu-rep")):
            continue
        raw = subprocess.run(["ncu", "-i", os.path.join(OUT, f), "--page", "raw", "--csv"],
                             capture_output=True, text=True).stdout
        rows = list(csv.reader(io.StringIO(raw)))
        if len(rows) < 3:
            continue
        hh = rows[0]
        if h is None:
            h, units = hh, rows[1]
        for r in rows[2:]:
            d = dict(zip(hh, r))
            n = short(d["Kernel Name"])
            if n in seen:
                continue
            seen.add(n)
            out.append([d.get(k, "") for k in h])
    return h, units, out


def ncu_top(tag):
    h, units, body = ncu_rows()
    if h is None:
        return
    rows = [h, units] + body
    want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
            "sm__throughput.avg.pct_of_peak_sustained_elapsed",
            "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
            "dram__throughput.avg.pct_of_peak_sustained_elapsed",
            "sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
            "sm__inst_executed_pipe_tc.avg.pct_of_peak_sustained_active",
            "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
            "smsp__warps_active.avg.pct_of_peak_sustained_active",
            "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
            "lts__t_sector_hit_rate.pct", "launch__registers_per_thread", "launch__grid_size"]
    idx = {w: h.index(w) for w in want if w in h}
    lines = [f"# {tag}: ncu --set full of the top kernels (c4 bench step)", "",
             "| kernel | " + " | ".join(w.split(".")[0] for w in idx) + " |",
             "|---|" + "---|" * len(idx)]
    traffic = {}
    for r in rows[2:]:
        n = short(r[h.index("Kernel Name")])
        vals = []
        for w, i in idx.items():
            vals.append(f"{r[i]} {units[i]}".strip())
        lines.append(f"| `{n}` | " + " | ".join(vals) + " |")
        try:
            rd = float(r[idx["dram__bytes_read.sum"]].replace(",", ""))
            wr = float(r[idx["dram__bytes_write.sum"]].replace(",", ""))
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
            rd *= scale.get(units[idx["dram__bytes_read.sum"]], 1)
            wr *= scale.get(units[idx["dram__bytes_write.sum"]], 1)
            base = n.split("<")[0].split("::")[-1]
            st = STAGE_OF.get(base)
            if st:
                traffic[f"{CONFIG_KEY}/{st}"] = rd + wr
        except (KeyError, ValueError):
            pass
    open(os.path.join(PROF, f"{tag}_ncu_top.md"), "w").write("\n".join(lines) + "\n")
    if traffic:
        json.dump({"source": f"profiles/{tag}_ncu_top.md", "dram_bytes_per_launch": traffic,
                   "note": "keys are <config name>-r<rank>/<stage> (the capture is of the c4 bench step); "
                           "a config that was not captured gets traffic null"},
                  open(os.path.join(PROF, "traffic.json"), "w"), indent=1)


def main():
    tag = sys.argv[1]
    os.makedirs(PROF, exist_ok=True)
    for f, dst in (("bench.json", f"{tag}_bench.json"), ("bench.err", f"{tag}_bench_stages.txt")):
        if os.path.exists(os.path.join(OUT, f)):
            shutil.copy(os.path.join(OUT, f), os.path.join(PROF, dst))
    launches(tag)
    ncu_top(tag)


if __name__ == "__main__":
    main()
