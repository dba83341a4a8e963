#!/usr/bin/env python
"""Instructions executed per OUTERMOST call site (the kernel-body line an inlined helper was
called from), from an ncu report and `nvdisasm -gi` of the same build.

    python tools/ncu_inline.py <report.ncu-rep|sass.csv.gz> <object.o> <ncu-name-substring> <mangled-substring> [top]
"""
import collections
import csv
import gzip
import io
import os
import re
import subprocess
import sys
import tempfile


def gi_lines(obj, mangled):
    d = tempfile.mkdtemp()
    subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(obj)], cwd=d, capture_output=True)
    cb = [os.path.join(d, f) for f in os.listdir(d) if f.endswith(".cubin")][0]
    txt = subprocess.run(["nvdisasm", "-gi", "-c", cb], capture_output=True, text=True).stdout
    out, cur, infn = [], None, False
    for ln in txt.splitlines():
        if ln.startswith("//----") and ".text." in ln:
            infn = mangled in ln
            continue
        if not infn:
            continue
        if "//## File" in ln:
            locs = re.findall(r'"([^"]+)", line (\d+)', ln)
            cur = (os.path.basename(locs[-1][0]), int(locs[-1][1]))   # outermost frame
            continue
        if re.search(r"/\*[0-9a-f]{4,}\*/", ln):
            out.append(cur)
    return out


def main():
    rep, obj, name, mangled = sys.argv[1:5]
    top = int(sys.argv[5]) if len(sys.argv) > 5 else 40
    if rep.endswith(".gz"):
        txt = gzip.open(rep, "rt").read()
    else:
        txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                             capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, blocks, cur = None, [], None
    for r in rows:
        if r and r[0] == "Kernel Name":
            cur = {"name": r[1], "rows": []}
            blocks.append(cur)
        elif r and r[0] == "Address":
            hdr = r
        elif cur is not None and hdr and len(r) >= len(hdr) - 1:
            cur["rows"].append(r)
    norm = lambda s: s.replace(" ", "").replace("(int)", "").replace("(bool)", "")
    b = next(x for x in blocks if name in norm(x["name"]))["rows"]
    ie = hdr.index("Instructions Executed")
    st = hdr.index("Warp Stall Sampling (All Samples)")
    f = lambda x: float(x.replace(",", "")) if x.replace(",", "").replace(".", "").isdigit() else 0.0
    locs = gi_lines(obj, mangled)
    if len(locs) != len(b):
        print(f"warning: {len(locs)} disassembled vs {len(b)} profiled", file=sys.stderr)
    agg = collections.defaultdict(lambda: [0.0, 0.0])
    for i in range(min(len(locs), len(b))):
        agg[locs[i]][0] += f(b[i][ie])
        agg[locs[i]][1] += f(b[i][st])
    ti = sum(a[0] for a in agg.values()) or 1
    ts = sum(a[1] for a in agg.values()) or 1
    print(f"total instructions {ti:.0f}")
    for k, a in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
        print(f"{str(k[0]) + ':' + str(k[1]) if k else '?':32s} inst {100 * a[0] / ti:6.2f}%  stall {100 * a[1] / ts:6.2f}%")


if __name__ == "__main__":
    main()
