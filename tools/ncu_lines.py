#!/usr/bin/env python
"""Aggregate an ncu SASS source page by CUDA source line.

    python tools/ncu_lines.py <report.ncu-rep> <object.o|.cubin> <ncu-name-substring> [top] [raw:<mangled-substring>]

Runs `ncu -i --page source --print-source sass --csv` and `nvdisasm -g` on the cubin of the
same build, matches instructions by order, and prints instructions executed and warp-stall
samples per (file, line) — the per-line view the ncu CSV export lacks.
"""
import collections
import csv
import io
import os
import re
import subprocess
import sys
import tempfile


def mangled_match(kernel, line):
    if kernel.startswith("raw:"):
        return kernel[4:] in line
    """kernel like 'k_resample_raw<1>' matches the mangled '14k_resample_rawILi1EE...'."""
    m = re.match(r"(\w+)(?:<([^>]*)>)?", kernel)
    name, targs = m.group(1), m.group(2)
    if name not in line:
        return False
    if targs is None:
        return True
    enc = ""
    for a in targs.split(","):
        a = a.strip()
        if a in ("true", "false"):
            enc += "Lb" + ("1" if a == "true" else "0") + "E"
        elif a.startswith("-"):
            enc += "Lin" + a[1:] + "E"
        else:
            enc += "Li" + a + "E"
    return f"{name}I{enc}" in line


def sass_lines(obj, kernel):
    d = tempfile.mkdtemp()
    if obj.endswith(".o") or obj.endswith(".so"):
        subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(obj)], cwd=d, capture_output=True)
        cubins = [os.path.join(d, f) for f in os.listdir(d) if f.endswith(".cubin")]
    else:
        cubins = [obj]
    out = []
    for cb in cubins:
        txt = subprocess.run(["nvdisasm", "-g", "-c", cb], capture_output=True, text=True).stdout
        cur = None
        infn = False
        for ln in txt.splitlines():
            if ln.startswith("//----") and ".text." in ln:
                infn = mangled_match(kernel, ln)
                continue
            if not infn:
                continue
            m = re.search(r'//## File "([^"]+)", line (\d+)', ln)
            if m:
                cur = (os.path.basename(m.group(1)), int(m.group(2)))
                continue
            if re.search(r"/\*[0-9a-f]{4,}\*/", ln):
                out.append((cur, ln.split("*/", 1)[1].strip()))
        if out:
            break
    return out


def main():
    rep, obj, kernel = sys.argv[1:4]
    top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
    mangled = sys.argv[5] if len(sys.argv) > 5 else kernel
    if rep.endswith(".csv.gz"):      # a saved `--page source --print-source sass --csv` export
        import gzip
        csvtxt = gzip.open(rep, "rt").read()
    else:
        csvtxt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                                capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(csvtxt)))
    hdr = None
    blocks, cur = [], None
    for r in rows:
        if r and r[0] == "Kernel Name":
            cur = {"name": r[1], "rows": []}
            blocks.append(cur)
        elif r and r[0] == "Address":
            hdr = r
        elif cur is not None and hdr and len(r) >= len(hdr) - 1:
            cur["rows"].append(r)
    blk = next(b for b in blocks if kernel in b["name"].replace(" ", "").replace("(int)", "").replace("(bool)", "").replace("true", "1").replace("false", "0"))
    ie, st, src = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Source")

    def f(x):
        try:
            return float(x.replace(",", ""))
        except ValueError:
            return 0.0

    lines = sass_lines(obj, mangled)
    n = min(len(lines), len(blk["rows"]))
    if len(lines) != len(blk["rows"]):
        print(f"warning: {len(lines)} disassembled vs {len(blk['rows'])} profiled instructions", file=sys.stderr)
    agg = collections.defaultdict(lambda: [0.0, 0.0, 0])
    for i in range(n):
        key = lines[i][0]
        a = agg[key]
        a[0] += f(blk["rows"][i][ie])
        a[1] += f(blk["rows"][i][st])
        a[2] += 1
    ti = sum(a[0] for a in agg.values())
    ts = sum(a[1] for a in agg.values())
    print(f"{'file:line':40s} {'inst%':>7s} {'stall%':>7s} {'#sass':>6s}")
    for key, a in sorted(agg.items(), key=lambda kv: -(kv[1][0] / ti + kv[1][1] / ts))[:top]:
        name = f"{key[0]}:{key[1]}" if key else "?"
        print(f"{name:40s} {100 * a[0] / ti:7.2f} {100 * a[1] / ts:7.2f} {a[2]:6d}")


if __name__ == "__main__":
    main()
