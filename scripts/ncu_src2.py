"""Per-source-line stall breakdown of one kernel from an ncu report (top stall columns).
    python scripts/ncu_src2.py <rep> <kernel-regex> <file-substring>"""
import csv, io, subprocess, sys
rep, kre, fsub = sys.argv[1:4]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "-k", f"regex:{kre}"], capture_output=True, text=True).stdout
cur = None; hdr = None; rows = []
for r in csv.reader(io.StringIO(out)):
    if len(r) >= 2 and r[0] == "File Path": cur = r[1]; continue
    if len(r) > 3 and r[0] == "Line No": hdr = r; continue
    if not hdr or not cur or fsub not in cur or len(r) < len(hdr): continue
    try: ln = int(r[0])
    except ValueError: continue
    d = dict(zip(hdr, r))
    def f(k):
        try: return float(d.get(k, 0) or 0)
        except ValueError: return 0.0
    tot = f("Warp Stall Sampling (All Samples)")
    if tot < 20: continue
    cols = {k[6:]: f(k) for k in hdr if k.startswith("stall_") and "Not Issued" not in k}
    top = sorted(cols.items(), key=lambda x: -x[1])[:4]
    print(f"L{ln:4d} {tot:6.0f} " + " ".join(f"{k}={v:.0f}" for k, v in top if v > 0) + f" | {r[1].strip()[:70]}")
