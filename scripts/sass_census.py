#!/usr/bin/env python
"""Per-kernel SASS opcode census of libttemb.so (cuobjdump -sass; no GPU needed).

    python scripts/sass_census.py [--out profiles/r02_sass_census.md]

Counts the opcodes that prove which hardware paths a kernel uses (B200_PROFILING.md):
UTCHMMA / UTCQMMA (tcgen05.mma), LDTM / STTM (TMEM ld / st), UTMALDG (tensor-map TMA load),
UBLKCP (1-D bulk copy), LDGSTS (Ampere cp.async), FFMA, FFMA2 (packed fp32 pairs), REDG, SHFL.
"""
from __future__ import annotations

import argparse
import collections
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_sc_wangwfmmd22_b200", "libttemb.so")
OPS = ["UTCHMMA", "UTCQMMA", "UTCBAR", "LDTM", "STTM", "UTMALDG", "UTMASTG", "UBLKCP", "LDGSTS", "SYNCS",
       "FFMA", "FFMA2", "REDG", "ATOMG", "SHFL", "LDS", "STS", "LDG", "STG"]


def demangle(name: str) -> str:
    try:
        return subprocess.run(["c++filt", name], capture_output=True, text=True).stdout.strip()
    except OSError:
        return name


def census(lib: str):
    txt = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-sass", lib], capture_output=True, text=True,
                         check=True).stdout
    kern = None
    counts = collections.OrderedDict()
    for line in txt.splitlines():
        m = re.match(r"\s*Function : (\S+)", line)
        if m:
            kern = demangle(m.group(1))
            kern = re.sub(r"^void ", "", kern)
            kern = re.sub(r"\((?!anonymous)[^()]*\)$", "", kern)
            kern = kern.replace("ttemb::(anonymous namespace)::", "").replace("ttemb::", "")
            counts.setdefault(kern, collections.Counter())
            continue
        m = re.match(r"\s*/\*[0-9a-f]{4,}\*/\s+(@!?U?P\w+\s+)?([A-Z][A-Z0-9_]*)(\.\S+)?", line)
        if m and kern is not None:
            op = m.group(2)
            for o in OPS:
                if op == o:
                    counts[kern][o] += 1
    return counts


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--lib", default=LIB)
    ap.add_argument("--out", default=None)
    a = ap.parse_args()
    c = census(a.lib)
    cols = [o for o in OPS if any(v[o] for v in c.values())]
    lines = ["| kernel | " + " | ".join(cols) + " |", "|---|" + "---|" * len(cols)]
    for k, v in c.items():
        lines.append(f"| `{k}` | " + " | ".join(str(v[o]) if v[o] else "" for o in cols) + " |")
    md = "\n".join(lines) + "\n"
    if a.out:
        with open(a.out, "w") as f:
            f.write("# SASS opcode census of libttemb.so (`python scripts/sass_census.py`)\n\n"
                    "Static instruction counts per kernel (cuobjdump -sass of the sm_100a build).  UTCHMMA = "
                    "tcgen05.mma, LDTM / STTM = tcgen05.ld / st, UTMALDG = tensor-map TMA load, UBLKCP = 1-D bulk "
                    "copy (cp.async.bulk), LDGSTS = cp.async (Ampere), REDG = global reductions.\n\n" + md)
    sys.stdout.write(md)


if __name__ == "__main__":
    main()
