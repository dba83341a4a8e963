#!/usr/bin/env python
"""Attribute an ncu SASS profile of one kernel to source-line ranges (phases), following
inlined call chains (nvdisasm -gi) to the outermost frame inside the chosen file.

    python tools/ncu_phases.py <report> <object.o> <ncu-name-substring> <raw:mangled> <file> a-b:name ...
"""
import collections, csv, io, os, re, subprocess, sys, tempfile

sys.path.insert(0, os.path.dirname(__file__))
import ncu_lines  # noqa: E402


def chains(obj, mangled):
    d = tempfile.mkdtemp()
    subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(obj)], cwd=d, capture_output=True)
    cb = [os.path.join(d, f) for f in os.listdir(d) if f.endswith(".cubin")][0]
    txt = subprocess.run(["nvdisasm", "-gi", "-c", cb], capture_output=True, text=True).stdout
    out, cur, infn, fresh = [], [], False, True
    for ln in txt.splitlines():
        if ln.startswith("//----") and ".text." in ln:
            infn = ncu_lines.mangled_match(mangled, ln)
            continue
        if not infn:
            continue
        if ln.strip().startswith("//## File"):
            if fresh:
                cur, fresh = [], False
            cur += re.findall(r'"([^"]+)", line (\d+)', ln)   # one inline level per line
            continue
        if re.search(r"/\*[0-9a-f]{4,}\*/", ln):
            fresh = True
            # innermost first, then the call sites outwards (deduplicated, order kept)
            seen, chain = set(), []
            for f, l in cur:
                if (f, l) not in seen:
                    seen.add((f, l))
                    chain.append((os.path.basename(f), int(l)))
            out.append(chain)
    return out


def main():
    rep, obj, name, mangled, fname = sys.argv[1:6]
    ranges = []
    for a in sys.argv[6:]:
        r, n = a.split(":")
        lo, hi = r.split("-")
        ranges.append((int(lo), int(hi), n))
    if rep.endswith(".csv.gz"):      # a saved `--page source --print-source sass --csv` export
        import gzip
        txt = gzip.open(rep, "rt").read()
    else:
        txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                             capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, blk, cur = None, None, None
    for r in rows:
        if r and r[0] == "Kernel Name":
            cur = name in r[1].replace(" ", "") and blk is None
            if cur:
                blk = []
        elif r and r[0] == "Address":
            hdr = r
        elif cur and hdr and len(r) >= len(hdr) - 1:
            blk.append(r)
    ie, st = hdr.index("Instructions Executed"), hdr.index("Warp Stall Sampling (All Samples)")
    ch = chains(obj, mangled)
    n = min(len(ch), len(blk))
    agg = collections.defaultdict(lambda: [0.0, 0.0])
    for i in range(n):
        lines = [l for f, l in ch[i] if f == fname]
        key = "other"
        # the outermost frame in a range marked '*' (kernel bodies) is used only when no other
        # range matches: device functions called from the body get their own phase
        for pref in (False, True):
            for l in reversed(lines):       # outermost first
                hit = [nm for lo, hi, nm in ranges if lo <= l <= hi and nm.endswith("*") == pref]
                if hit:
                    key = hit[0]
                    break
            if key != "other":
                break
        a = agg[key]
        a[0] += float(blk[i][ie] or 0)
        a[1] += float(blk[i][st] or 0)
    ti = sum(a[0] for a in agg.values()) or 1
    ts = sum(a[1] for a in agg.values()) or 1
    for k, a in sorted(agg.items(), key=lambda kv: -kv[1][0]):
        print(f"{k:24s} inst {100 * a[0] / ti:6.2f}%  stall {100 * a[1] / ts:6.2f}%")


if __name__ == "__main__":
    main()
