#!/usr/bin/env python
"""Turn a scripts/evidence.sh run (gpurun_out/<tag>_*) into committed evidence under profiles/.

    python tools/summarize_profiles.py <tag> [round]      # e.g. r02a r02

Writes profiles/<round>_bench_<config>.json, profiles/<round>_launches_<config>.csv,
profiles/<round>_ncu_summary.md (per-kernel metrics incl. the FMA/ALU pipe utilisation, the ALU
roofline of the blur/conversion-bound kernels) and profiles/ncu_traffic.json (DRAM bytes per
launch of each config's dominant kernel, read by bench.py for the roofline "traffic" field).
"""
import csv
import glob
import gzip
import io
import json
import os
import shutil
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")

METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput % of peak"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %"),
    ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue active %"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "achieved occupancy %"),
    ("smsp__inst_executed.sum", "warp instructions"),
    ("launch__registers_per_thread", "registers/thread"),
    ("launch__shared_mem_per_block_dynamic", "dynamic smem/block"),
    ("launch__grid_size", "grid"),
    ("launch__block_size", "block"),
    ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "tensor pipe %"),
    ("sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", "FMA pipe inst %"),
    ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "FMA pipe cycles %"),
    ("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active", "ALU pipe inst %"),
    ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "LSU pipe inst %"),
]


def to_bytes(v, unit):
    f = float(v.replace(",", ""))
    return f * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)


def raw_rows(path):
    rows = list(csv.reader(open(path)))
    if len(rows) < 3:
        return [], [], []
    return rows[0], rows[1], rows[2:]


def main():
    tag = sys.argv[1] if len(sys.argv) > 1 else "r02a"
    rnd = sys.argv[2] if len(sys.argv) > 2 else tag[:3]
    os.makedirs(PROF, exist_ok=True)
    traffic = {}
    md = [f"# ncu summary, round {rnd}", "",
          "Captured with `scripts/evidence.sh` on one B200 (`ncu --set full --clock-control none`, "
          "kernels matching `k_(plain|stream|stencil|direct|copy)`, 2 launches after 6 skipped). Per-launch, "
          "cold-cache, serialised: compare shares, not absolutes. Bench numbers come from "
          "`bench.py` (CUDA events, no profiler).", ""]
    for path in sorted(glob.glob(os.path.join(OUT, f"{tag}_ncu_raw_*.csv"))):
        cfg = os.path.basename(path)[len(f"{tag}_ncu_raw_"):-4]
        hdr, units, data = raw_rows(path)
        if not data:
            continue
        md += [f"## {cfg}", "", "| kernel | " + " | ".join(m[1] for m in METRICS) + " |",
               "|---" * (len(METRICS) + 1) + "|"]
        per_kernel = {}
        for d in data:
            name = d[hdr.index("Kernel Name")].split("(")[0]
            vals = []
            for m, _ in METRICS:
                if m in hdr:
                    i = hdr.index(m)
                    vals.append(f"{d[i]} {units[i]}".strip())
                else:
                    vals.append("-")
            md.append(f"| `{name}` | " + " | ".join(vals) + " |")
            dur = float(d[hdr.index("gpu__time_duration.sum")].replace(",", ""))
            dram = to_bytes(d[hdr.index("dram__bytes_read.sum")], units[hdr.index("dram__bytes_read.sum")]) + \
                to_bytes(d[hdr.index("dram__bytes_write.sum")], units[hdr.index("dram__bytes_write.sum")])
            k = per_kernel.setdefault(name, [0.0, 0.0, 0])
            k[0] += dur
            k[1] += dram
            k[2] += 1
        md.append("")
        dom = max(per_kernel.items(), key=lambda kv: kv[1][0])
        traffic[cfg] = {"kernel": dom[0], "dram_bytes_per_launch": dom[1][1] / dom[1][2],
                        "ncu_duration_per_launch": dom[1][0] / dom[1][2],
                        "source": f"profiles/{rnd}_ncu_summary.md"}
        # instruction counts and pipe utilisation of the dominant kernel (the ALU roofline)
        for d in data:
            if d[hdr.index("Kernel Name")].split("(")[0] != dom[0]:
                continue
            def val(m):
                return float(d[hdr.index(m)].replace(",", "")) if m in hdr and d[hdr.index(m)] else None
            traffic[cfg].update({
                "warp_inst_per_launch": val("smsp__inst_executed.sum"),
                "alu_pipe_pct": val("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active"),
                "fma_pipe_pct": val("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active"),
                "issue_active_pct": val("smsp__issue_active.avg.pct_of_peak_sustained_active")})
            break
        det = os.path.join(OUT, f"{tag}_ncu_details_{cfg}.csv")
        if os.path.exists(det):
            notes = []
            for r in csv.reader(open(det)):
                if len(r) > 15 and r[12] in ("IssueSlotUtilization", "CPIStall", "TheoreticalOccupancy") and r[14]:
                    notes.append(f"- {r[4].split('(')[0]} / {r[12]}: {r[14][:300]}")
            md += sorted(set(notes))[:6] + [""]
    for path in sorted(glob.glob(os.path.join(OUT, f"{tag}_launches_*.csv"))):
        cfg = os.path.basename(path)[len(f"{tag}_launches_"):-4]
        rows = [r for r in csv.reader(open(path)) if len(r) > 10]
        if rows:
            with open(os.path.join(PROF, f"{rnd}_launches_{cfg}.csv"), "w", newline="") as f:
                csv.writer(f).writerows(rows)
    for path in sorted(glob.glob(os.path.join(OUT, f"{tag}_bench_*.json"))):
        name = os.path.basename(path)[len(f"{tag}_bench_"):-5]
        try:
            line = json.loads(open(path).read().strip().splitlines()[-1])
        except (ValueError, IndexError):
            continue
        json.dump(line, open(os.path.join(PROF, f"{rnd}_bench_{name}.json"), "w"), indent=1)
    open(os.path.join(PROF, f"{rnd}_ncu_summary.md"), "w").write("\n".join(md) + "\n")
    json.dump(traffic, open(os.path.join(PROF, "ncu_traffic.json"), "w"), indent=1)
    for f in ("gpu.txt", "pytest_gpu.log", "smoke.log"):
        if os.path.exists(os.path.join(OUT, f"{tag}_{f}")):
            shutil.copy(os.path.join(OUT, f"{tag}_{f}"), os.path.join(PROF, f"{rnd}_{f}"))
    for path in sorted(glob.glob(os.path.join(OUT, f"{tag}_ncu_sass_*.csv.gz"))):
        shutil.copy(path, os.path.join(PROF, os.path.basename(path).replace(tag, rnd)))
    print(open(os.path.join(PROF, f"{rnd}_ncu_summary.md")).read())
    print(json.dumps(traffic, indent=1))


if __name__ == "__main__":
    main()
