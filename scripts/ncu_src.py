"""Per-source-line table (samples, instructions executed, smem wavefronts) of one kernel.
    python scripts/ncu_src.py <rep> <kernel-regex> <file-substring> [lo hi]"""
import csv, io, subprocess, sys
rep, kre, fsub = sys.argv[1:4]
lo, hi = (int(sys.argv[4]), int(sys.argv[5])) if len(sys.argv) > 5 else (0, 10**9)
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "-k", f"regex:{kre}"], capture_output=True, text=True).stdout
cur = None; hdr = None
for r in csv.reader(io.StringIO(out)):
    if len(r) >= 2 and r[0] == "File Path": cur = r[1]; continue
    if len(r) > 3 and r[0] == "Line No": hdr = r; continue
    if not hdr or not cur or fsub not in cur or len(r) < len(hdr): continue
    try: ln = int(r[0])
    except ValueError: continue
    if not (lo <= ln <= hi): continue
    d = dict(zip(hdr, r))
    s, ie = d.get("Warp Stall Sampling (All Samples)", "0"), d.get("Instructions Executed", "0")
    wf = d.get("L1 Wavefronts Shared", "0")
    if s in ("0", "") and ie in ("0", ""): continue
    print(f"L{ln:4d} samp {s:>6} inst {ie:>9} smemwf {wf:>8} | {r[1].strip()[:80]}")
