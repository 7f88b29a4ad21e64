"""Summarise the config sweep (scripts/config_sweep.sh) into profiles/<tag>_config_sweep.md.

    python scripts/summarize_sweep.py <round-tag>

Copies gpurun_out/sweep/*.json to profiles/<tag>_config_sweep/ and writes the table.
"""
import glob
import json
import os
import shutil
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = """# {tag}: bench lines of every BASELINE config (one B200, `scripts/config_sweep.sh`)

Parity of every config against the oracle: tests/test_gpu_parity.py (c1-c3 full batch; c4 full batch fwd + bwd + fused SGD / Adagrad; c5 r32/r64/r128 full-size sampled fwd + bwd).
tcgen05 path: c2 (R = 16 stored zero-padded to 32, DESIGN.md R28), c3 and c5-r32 (native R = 32), c4 and c5-r64 (R = 64), c5-r128 (R = 128); FFMA path: c1 (R = 8).

| workload | tables | dim | R | batch | L | opt | ms/step | lookups/s | e2e lookups/s |
|---|---|---|---|---|---|---|---|---|---|
"""


def main(tag):
    src = os.path.join(ROOT, "gpurun_out", "sweep")
    dst = os.path.join(ROOT, "profiles", f"{tag}_config_sweep")
    os.makedirs(dst, exist_ok=True)
    rows = []
    for f in sorted(glob.glob(os.path.join(src, "*.json"))):
        try:
            d = json.loads(open(f).read().strip().splitlines()[-1])
        except (ValueError, IndexError):
            print("skip (no JSON line):", f)
            continue
        shutil.copy(f, dst)
        c = d["config"]
        e2e = d.get("e2e") or {}
        rows.append("| {} | {} | {} | {} | {} | {} | {} | {:.3f} | {:.1f} M | {} |".format(
            c["workload"], c.get("tables"), c.get("dim"), c.get("tt_rank"), c.get("batch_per_gpu"),
            c.get("pooling"), c.get("optimizer"), d["ms_per_step"], d["value"] / 1e6,
            f"{e2e['value'] / 1e6:.1f} M" if e2e.get("value") else "-"))
    out = os.path.join(ROOT, "profiles", f"{tag}_config_sweep.md")
    open(out, "w").write(HEADER.format(tag=tag) + "\n".join(sorted(rows)) + "\n")
    print(out)


if __name__ == "__main__":
    main(sys.argv[1])
