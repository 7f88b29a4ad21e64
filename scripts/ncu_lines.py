"""Rank CUDA source lines of one kernel in an ncu report by warp-stall samples.

    python scripts/ncu_lines.py gpurun_out/prof.ncu-rep <kernel-regex> [top]
"""
import csv
import io
import re
import subprocess
import sys

rep, kre = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass", "-k", "regex:" + (sys.argv[4] if len(sys.argv) > 4 else ".")],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = None
fname = func = ""
lines = {}
for r in rows:
    if len(r) == 2 and r[0] in ("File Path", "File Name"):
        fname = r[1].split("/")[-1]
        continue
    if len(r) == 2 and r[0] == "Function Name":
        func = r[1]
        continue
    if r and r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) < 5 or not r[0].isdigit() or not re.search(kre, func):
        continue
    key = (func, fname, int(r[0]))
    cur = lines.setdefault(key, {"src": r[1].strip(), "samples": 0, "stalls": {}})
    try:
        cur["samples"] += int(r[hdr.index("Warp Stall Sampling (All Samples)")])
    except Exception:
        pass
    for i, h in enumerate(hdr):
        if h.startswith("stall_") and "Not Issued" not in h and i < len(r):
            try:
                v = int(r[i])
            except Exception:
                continue
            if v:
                cur["stalls"][h] = cur["stalls"].get(h, 0) + v
tot = sum(v["samples"] for v in lines.values()) or 1
print(f"total samples {tot}")
for (fn, f, ln), v in sorted(lines.items(), key=lambda kv: -kv[1]["samples"])[:top]:
    st = sorted(v["stalls"].items(), key=lambda kv: -kv[1])[:3]
    print(f"{100 * v['samples'] / tot:5.1f}% {f}:{ln:<4} {v['src'][:60]:60s} {st}")
