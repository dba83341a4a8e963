#!/usr/bin/env python
"""Key metrics of one kernel from an `ncu --page raw --csv` export plus its executed-instruction
basic blocks from the SASS source page (both saved by scripts/gpu_iter.sh).

    python tools/ncu_summary.py <raw.csv> [sass.csv.gz] [values-per-launch]
"""
import csv
import gzip
import io
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "launch__block_size", "sm__inst_executed.sum",
        "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active"]


def raw(path):
    rows = list(csv.reader(open(path)))
    hdr, units = rows[0], rows[1]
    for vals in rows[2:]:
        yield {h: (v, u) for h, v, u in zip(hdr, vals, units)}


def main():
    for d in raw(sys.argv[1]):
        print(d.get("Kernel Name", ("?",))[0][:90])
        for k in KEYS:
            if k in d:
                print(f"  {k:70s} {d[k][0]:>14s} {d[k][1]}")
        st = {k.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", ""): float(v[0])
              for k, v in d.items() if k.startswith("smsp__average_warps_issue_stalled_") and
              k.endswith("per_issue_active.ratio") and v[0] not in ("", "n/a")}
        print("  stalls/issue:", ", ".join(f"{k} {v:.2f}" for k, v in sorted(st.items(), key=lambda kv: -kv[1]) if v > 0.1))
    if len(sys.argv) > 2:
        rows = list(csv.reader(io.StringIO(gzip.open(sys.argv[2], "rt").read())))
        hdr, cur, blocks = None, None, []
        for r in rows:
            if r and r[0] == "Kernel Name":
                cur = []
                blocks.append(cur)
            elif r and r[0] == "Address":
                hdr = r
            elif cur is not None and hdr and len(r) >= len(hdr) - 1:
                cur.append(r)
        ie, src, th = hdr.index("Instructions Executed"), hdr.index("Source"), hdr.index("Thread Instructions Executed")
        segs = []
        for r in blocks[0]:
            n = float(r[ie].replace(",", "") or 0)
            t = float(r[th].replace(",", "") or 0)
            if segs and segs[-1][0] == n:
                segs[-1][1] += 1
                segs[-1][2] += t
                segs[-1][4] = r[src].strip()[:44]
            else:
                segs.append([n, 1, t, r[src].strip()[:44], r[src].strip()[:44]])
        tot = sum(s[0] * s[1] for s in segs)
        vals = float(sys.argv[3]) if len(sys.argv) > 3 else 0
        print(f"  warp instructions {tot:.0f}" + (f", lane instructions per value {32 * tot / vals:.2f}" if vals else ""))
        for s in sorted(segs, key=lambda s: -s[0] * s[1])[:18]:
            print(f"  {s[0] / 1e3:8.1f}K x {s[1]:3d} = {100 * s[0] * s[1] / tot:5.2f}%  lanes {s[2] / max(1, s[0] * s[1]):4.1f}  "
                  f"{s[3]} .. {s[4]}")


if __name__ == "__main__":
    main()
