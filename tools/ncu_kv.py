#!/usr/bin/env python
"""Key ncu details-page metrics per kernel of a report: python tools/ncu_kv.py <report.ncu-rep>"""
import csv
import io
import subprocess
import sys

KEYS = ('Duration', 'DRAM Throughput', 'Compute (SM) Throughput', 'Issue Slots Busy', 'Achieved Occupancy',
        'Executed Instructions', 'Registers Per Thread', 'Dynamic Shared Memory Per Block', 'Grid Size',
        'Block Size', 'Theoretical Occupancy', 'No Eligible', 'Active Warps Per Scheduler',
        'Eligible Warps Per Scheduler', 'Warp Cycles Per Issued Instruction', 'L1/TEX Hit Rate', 'L2 Hit Rate',
        'Memory Throughput', 'Mem Busy')
txt = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "details", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
h = rows[0]
for r in rows[1:]:
    d = dict(zip(h, r))
    if d.get('Metric Name') in KEYS:
        print(d['ID'], d['Kernel Name'][:34], '|', d['Metric Name'], d['Metric Value'], d['Metric Unit'])
