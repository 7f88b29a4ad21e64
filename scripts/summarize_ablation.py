"""profiles/<tag>_ablation.md from gpurun_out/abl/*.json (scripts/ablation.sh): the paper's
optimisation-breakdown toggles (Fig. 14/17/18) and the paper-design comparator."""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ABL = os.path.join(ROOT, "gpurun_out", "abl")
tag = sys.argv[1]
PAPER = {"no_reuse": "1.75x lookup from reuse (Fig. 17); -10 % throughput (Fig. 14)",
         "no_agg": "1.40x backward from aggregation (Fig. 18); -52 % throughput (Fig. 14)",
         "unfused": "1.15x backward from the fused update (Fig. 18)",
         "perm": "index reordering: 1.05x lookup, 1.06x backward, -13 % throughput",
         "perm_bij": "(runtime bijection restores part of the reordering gain)",
         "paper": "the paper's design: Alg. 1 reuse + cuBLAS batched GEMM (P:346)",
         "hybrid": "hybrid placement (P:310): tables <= 1M rows kept dense (speed-up, not a slowdown)"}
lines = [f"# {tag}: optimisation breakdown on B200 (scripts/ablation.sh)", "",
         "One B200, `bench.py --steps 10 --warmup 3` (CUDA-graph replay, L2 flushed between steps); "
         "`--impl paper` = comparators/paper_design.py (torch + cuBLAS fp32, eager), 5 steps.",
         "slowdown = variant ms / base ms.  Every variant is parity-tested against the oracle "
         "(tests/test_gpu_parity.py::test_ablation_switches, ::test_runtime_bijection, "
         "tests/test_paper_comparator.py).", ""]
for cfg in ("c4", "c3", "c2"):
    base_p = os.path.join(ABL, f"{cfg}-base.json")
    if not os.path.exists(base_p):
        continue
    base = json.load(open(base_p))
    lines += [f"## {cfg} ({base['config']['workload']})", "",
              "| variant | ms/step | lookups/s | slowdown vs ours | U | P | paper's figure |",
              "|---|---|---|---|---|---|---|"]
    for v in ("base", "no_reuse", "no_agg", "unfused", "perm", "perm_bij", "paper", "hybrid"):
        p = os.path.join(ABL, f"{cfg}-{v}.json")
        if not os.path.exists(p):
            continue
        try:
            d = json.load(open(p))
        except json.JSONDecodeError:
            continue
        sr = d.get("step_roofline", {})
        lines.append(f"| {v} | {d['ms_per_step']:.3f} | {d['value'] / 1e6:.1f} M | "
                     f"{d['ms_per_step'] / base['ms_per_step']:.2f}x | {sr.get('U', '')} | {sr.get('P', '')} | "
                     f"{PAPER.get(v, '')} |")
    lines.append("")
open(os.path.join(ROOT, "profiles", f"{tag}_ablation.md"), "w").write("\n".join(lines) + "\n")
print("\n".join(lines))
