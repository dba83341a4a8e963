#!/usr/bin/env python
"""Hot straight-line SASS blocks of one kernel in an ncu report, with source lines.

    python tools/ncu_blocks.py <report> <object.o> <ncu-name-substring> <raw:mangled-substring> [top]
"""
import csv
import io
import subprocess
import sys

sys.path.insert(0, __import__("os").path.dirname(__file__))
import ncu_lines  # noqa: E402


def main():
    rep, obj, name, mangled = sys.argv[1:5]
    top = int(sys.argv[5]) if len(sys.argv) > 5 else 25
    txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    blocks, cur, hdr = [], None, None
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
    ie, src = hdr.index("Instructions Executed"), hdr.index("Source")

    def f(x):
        try:
            return float(x.replace(",", ""))
        except ValueError:
            return 0.0

    lines = ncu_lines.sass_lines(obj, mangled)
    tot = sum(f(r[ie]) for r in b)
    out, prev, start, acc = [], None, 0, 0.0
    for i, r in enumerate(b):
        c = f(r[ie])
        if c != prev:
            if prev:
                out.append((start, i - 1, prev, acc))
            prev, start, acc = c, i, 0.0
        acc += c
    if prev:
        out.append((start, len(b) - 1, prev, acc))
    out.sort(key=lambda x: -x[3])
    print(f"total warp instructions {tot:.0f}")
    for s, e, c, a in out[:top]:
        ln = sorted({l[0][1] for l in lines[s:e + 1] if l[0]}) if len(lines) == len(b) else []
        print(f"[{s:5d}-{e:5d}] n={e - s + 1:4d} exec={c:9.0f} share={100 * a / tot:5.1f}% lines={ln[:10]} "
              f"first={b[s][src].strip()[:40]}")


if __name__ == "__main__":
    main()
