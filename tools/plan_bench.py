#!/usr/bin/env python
"""Compile and run tools/plan_bench.cpp (host-only epoch-planner timing) against libsand.so."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_sosp_yelllhkh25_b200")
OUT = os.path.join(PKG, "build", "plan_bench")
cmd = ["g++", "-O2", "-std=c++17", "-I", os.path.join(ROOT, "include"), "-I", os.path.join(PKG, "csrc"),
       "-I", "/usr/local/cuda/include", os.path.join(ROOT, "tools", "plan_bench.cpp"), "-L", PKG, "-lsand",
       "-L", "/usr/local/cuda/lib64", "-lcudart", f"-Wl,-rpath,{PKG}", "-o", OUT]
subprocess.check_call(cmd)
for cfg in (sys.argv[1:] or ["k400", "slowfast"]):
    subprocess.check_call([OUT, cfg])
