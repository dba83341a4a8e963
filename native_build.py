"""Native build for the repo: the product library, the oracle and the input generator.

Everything is compiled in-tree (the .so files travel to the GPU box with the
gpurun snapshot). CUDA code targets sm_100a only:
``-gencode arch=compute_100a,code=sm_100a -lineinfo``.

    python native_build.py            # build all
    python native_build.py product    # only libsand.so
"""
from __future__ import annotations

import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.abspath(__file__))
PKG = os.path.join(ROOT, "paper_conf_sosp_yelllhkh25_b200")
CSRC = os.path.join(PKG, "csrc")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
CUDA_HOME = os.environ.get("CUDA_HOME", "/usr/local/cuda")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _run(cmd):
    print(" ".join(cmd), flush=True)
    subprocess.run(cmd, check=True, cwd=ROOT)


def _run_parallel(cmds):
    """Compile the kernel units concurrently (each nvcc is single-threaded)."""
    from concurrent.futures import ThreadPoolExecutor
    for c in cmds:
        print(" ".join(c), flush=True)

    def one(c):
        r = subprocess.run(c, cwd=ROOT, capture_output=True, text=True)
        return c, r

    with ThreadPoolExecutor(max_workers=max(1, min(len(cmds), os.cpu_count() or 1))) as ex:
        results = list(ex.map(one, cmds))
    for c, r in results:
        sys.stdout.write(r.stdout)
        sys.stderr.write(r.stderr)
        if r.returncode != 0:
            raise subprocess.CalledProcessError(r.returncode, c)


def _stale(target, sources):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(s) > t for s in sources)


def build_synth(force=False):
    d = os.path.join(ROOT, "synth")
    hdr = os.path.join(d, "nv12_synth.h")
    host_src = os.path.join(d, "synth.c")
    host_so = os.path.join(d, "libsynth_host.so")
    if force or _stale(host_so, [host_src, hdr]):
        _run(["gcc", "-O2", "-std=c11", "-shared", "-fPIC", host_src, "-o", host_so])
    cu_src = os.path.join(d, "synth_cuda.cu")
    cu_so = os.path.join(d, "libsynth_cuda.so")
    if force or _stale(cu_so, [cu_src, hdr]):
        _run([NVCC, *ARCH, "-O3", "-lineinfo", "-shared", "-Xcompiler", "-fPIC", cu_src, "-o", cu_so])


def build_oracle(force=False):
    src = os.path.join(ROOT, "oracle", "sand_oracle.c")
    so = os.path.join(ROOT, "oracle", "libsand_oracle.so")
    if force or _stale(so, [src]):
        # plain C, no contraction, no fast-math: every fp op is a correctly rounded basic op or fmaf
        _run(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-shared", "-fPIC",
              src, "-o", so, "-lm"])


PRODUCT_CPP = ["sand_api.cpp", "store.cpp", "planner.cpp", "view.cpp", "objcache.cpp"]
PRODUCT_CU = ["materialize.cu", "store_kernels.cu", "mat_plain.cu", "mat_stream.cu", "mat_direct.cu",
              "mat_stencil.cu", "mat_crop.cu"]
PRODUCT_HDR = ["internal.h", "plan_types.h", "planner.h", "kernels.h", "kernels_common.cuh", "k_resample.cuh",
               "k_stream.cuh", "k_plain.cuh", "k_stencil.cuh", "k_direct.cuh", "k_copy.cuh", "k_crop.cuh"]


def build_product(force=False, variant=None, defines=()):
    """libsand.so, or libsand_<variant>.so compiled with extra -D defines (A/B experiments)."""
    if variant:
        import shutil
        bdir = os.path.join(PKG, "build_" + variant)
        os.makedirs(bdir, exist_ok=True)
        objs = []
        inc = ["-I", os.path.join(ROOT, "include"), "-I", CSRC]
        jobs = []
        for s in PRODUCT_CPP:   # host units too: the defines may change shared headers
            obj = os.path.join(bdir, s + ".o")
            objs.append(obj)
            jobs.append(["g++", "-O2", "-std=c++17", "-fPIC", "-ffp-contract=off", "-fno-fast-math", "-Wall",
                         "-I", os.path.join(CUDA_HOME, "include"), *["-D" + d for d in defines], *inc, "-c",
                         os.path.join(CSRC, s), "-o", obj])
        for s in PRODUCT_CU:
            obj = os.path.join(bdir, s + ".o")
            objs.append(obj)
            jobs.append([NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xptxas", "-v",
                         "--expt-relaxed-constexpr", *["-D" + d for d in defines], *inc, "-c", os.path.join(CSRC, s),
                         "-o", obj])
        _run_parallel(jobs)
        _run([NVCC, *ARCH, "-shared", "-Xcompiler", "-fPIC", *objs, "-o", os.path.join(PKG, f"libsand_{variant}.so"),
              "-lcudart", "-lpthread"])
        return
    os.makedirs(os.path.join(PKG, "build"), exist_ok=True)
    inc = ["-I", os.path.join(ROOT, "include"), "-I", CSRC]
    hdrs = [os.path.join(ROOT, "include", "sand.h")] + [os.path.join(CSRC, h) for h in PRODUCT_HDR]
    objs = []
    for s in PRODUCT_CPP:
        src = os.path.join(CSRC, s)
        obj = os.path.join(PKG, "build", s + ".o")
        objs.append(obj)
        if force or _stale(obj, [src] + hdrs):
            # host planner: IEEE double, no contraction (R#20 bit-exactness discipline)
            _run(["g++", "-O2", "-std=c++17", "-fPIC", "-ffp-contract=off", "-fno-fast-math", "-Wall",
                  "-I", os.path.join(CUDA_HOME, "include"), *inc, "-c", src, "-o", obj])
    jobs = []
    for s in PRODUCT_CU:
        src = os.path.join(CSRC, s)
        obj = os.path.join(PKG, "build", s + ".o")
        objs.append(obj)
        if force or _stale(obj, [src] + hdrs):
            jobs.append([NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC",
                         "-Xptxas", "-v", "--expt-relaxed-constexpr", *inc, "-c", src, "-o", obj])
    _run_parallel(jobs)
    so = os.path.join(PKG, "libsand.so")
    if force or _stale(so, objs):
        _run([NVCC, *ARCH, "-shared", "-Xcompiler", "-fPIC", *objs, "-o", so, "-lcudart", "-lpthread"])


def build_all(force=False):
    build_synth(force)
    build_oracle(force)
    build_product(force)


if __name__ == "__main__":
    what = sys.argv[1:] or ["all"]
    force = "--force" in what
    what = [w for w in what if w != "--force"] or ["all"]
    if what and what[0] == "variant":   # python native_build.py variant <name> DEF=1 ...
        build_product(variant=what[1], defines=what[2:])
        sys.exit(0)
    for w in what:
        {"all": build_all, "synth": build_synth, "oracle": build_oracle, "product": build_product}[w](force)
