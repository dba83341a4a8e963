#!/usr/bin/env python
"""Executed-instruction mix of one kernel from a saved ncu SASS source page.

    python tools/sass_mix.py <sass.csv.gz> [kernel-substring] [full]

Prints the share of executed warp instructions per opcode (and per full opcode with
modifiers when `full` is given), the total, and lane instructions per output value
when SAND_VALUES (output values per launch) is set in the environment.
"""
import collections
import csv
import gzip
import io
import os
import re
import sys


def load(path, kernel=None):
    rows = list(csv.reader(io.StringIO(gzip.open(path, "rt").read())))
    hdr, blocks, cur = None, [], None
    for r in rows:
        if r and r[0] == "Kernel Name":
            cur = {"name": r[1], "rows": []}
            blocks.append(cur)
        elif r and r[0] == "Address":
            hdr = r
        elif cur is not None and hdr and len(r) >= len(hdr) - 1:
            cur["rows"].append(r)
    b = next(b for b in blocks if kernel is None or kernel in b["name"])
    return hdr, b


def main():
    path = sys.argv[1]
    kernel = sys.argv[2] if len(sys.argv) > 2 and sys.argv[2] != "-" else None
    full = len(sys.argv) > 3
    hdr, b = load(path, kernel)
    ie, src = hdr.index("Instructions Executed"), hdr.index("Source")
    ops, tot = collections.Counter(), 0.0
    for r in b["rows"]:
        n = float(r[ie].replace(",", "") or 0)
        tot += n
        s = re.sub(r"^@!?U?P\w+\s+", "", r[src].strip())
        op = s.split()[0] if s else "?"
        ops[op if full else op.split(".")[0]] += n
    print(b["name"][:100])
    for k, v in ops.most_common(60):
        print(f"{k:28s} {100 * v / tot:6.2f}")
    vals = float(os.environ.get("SAND_VALUES", "0"))
    print(f"total warp instructions {tot:.0f}" + (f"  lane instr/value {32 * tot / vals:.2f}" if vals else ""))


if __name__ == "__main__":
    main()
