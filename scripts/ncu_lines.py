"""Rank CUDA source lines of one kernel in an ncu report by warp-stall samples.

    python scripts/ncu_lines.py gpurun_out/prof.ncu-rep <kernel-regex> [top]
"""
import csv
import io
import subprocess
import sys

rep, kre = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "-k", f"regex:{kre}"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hdr = None
lines = []
cur = None
for r in rows:
    if len(r) > 4 and r[0] == "Line No":
        hdr = r
        continue
    if hdr is None or len(r) < 5:
        continue
    if r[0]:
        cur = {"line": r[0], "src": r[1].strip(), "samples": 0, "stalls": {}}
        lines.append(cur)
        try:
            cur["samples"] = int(r[hdr.index("Warp Stall Sampling (All Samples)")])
        except Exception:
            pass
        for i, h in enumerate(hdr):
            if h.startswith("stall_") and i < len(r):
                try:
                    v = int(r[i])
                except Exception:
                    continue
                if v:
                    cur["stalls"][h] = cur["stalls"].get(h, 0) + v
tot = sum(l["samples"] for l in lines) or 1
for l in sorted(lines, key=lambda x: -x["samples"])[:top]:
    st = sorted(l["stalls"].items(), key=lambda kv: -kv[1])[:3]
    print(f"{100*l['samples']/tot:5.1f}% L{l['line']:>4} {l['src'][:70]:70s} {st}")
