#!/usr/bin/env python
"""Benchmark of the per-batch view materialisation path (BASELINE.json metric:
output frames/s per GPU & box at 1/2/4/8 B200; HBM GB/s vs peak).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config k400] [--impl sand|reference]
    torchrun --nproc-per-node N --master-addr 127.0.0.1 bench.py --gpus N ...

A step = one read_batch (all §8(a) rows) of one batch per rank. Inputs are
resident in HBM (a replicated synthetic store per GPU, far larger than L2) when
the timed region starts; the timed region is bracketed by barrier +
synchronize, timed with CUDA events on the read stream, max over ranks. Rank 0
prints ONE JSON line. `--impl reference` times the CPU oracle (the reference
arm for this paper: SAND's own engine is CPU code) on the same config.
"""
from __future__ import annotations

import argparse
import gc
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

DEFAULT_STEPS = {"tiny": 2000, "k400": 3000, "slowfast": 3000, "twoview": 1000, "ray": 1000, "slowfast_hd": 1000}


def log(*a):
    print(*a, file=sys.stderr, flush=True)


def dist_env():
    rank = int(os.environ.get("RANK", "0"))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return rank, world, local


# ------------------------------------------------------------------ clocks (nvidia-smi during the timed region)
class ClockSampler:
    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, device: int):
        self.device = device
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.device), f"--query-gpu={self.FIELDS}", "--format=csv,noheader,nounits",
                 "-lms", "20"], stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except OSError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.05)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=5)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm, smax, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                smax.append(float(parts[1]))
            except ValueError:
                continue
            for n, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        sm.sort()
        return {"sm_mhz": sm[len(sm) // 2] if sm else None, "sm_max_mhz": max(smax) if smax else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ------------------------------------------------------------------ peaks
def measured_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy read+write)"
    return 6650.0, "fallback (B200_PROFILING.md 6.65 TB/s)"


# kernel of each item class (SAND_N_CLASSES: mild plain, heavy plain, rotation/blur); the roofline's
# subject is the class with the most kernel time, its bytes / its own event-timed duration
# kernel of each item class (plain mild, heavy, stencil) per config: the mild class runs k_plainw
# (k_plain only for views wider than 256 / spans beyond 384 px), identity-scale batches k_copy
CLASS_KERNELS = {"slowfast": ("k_copy", "k_direct", "k_stencil2")}
DEFAULT_CLASS_KERNELS = ("k_plainw", "k_direct", "k_stencil2")


def ncu_record(config: str):
    """The committed ncu --set full record of a config's dominant kernel (profiles/ncu_traffic.json)."""
    p = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    if os.path.exists(p):
        return json.load(open(p)).get(config)
    return None


def ncu_traffic(config: str):
    """DRAM bytes per launch of the dominant kernel from the committed ncu --set full summary."""
    r = ncu_record(config)
    return r.get("dram_bytes_per_launch") if r else None


def alu_roofline(config, per_class, sm_count, clock_mhz):
    """Instruction-issue roofline of the dominant kernel: its warp instructions per
    launch (ncu) over its own event-timed duration, against the issue peak of one warp
    instruction per SM sub-partition per clock (148 SMs x 4 x clock); with the ALU pipe's share."""
    r = ncu_record(config)
    if not r or not r.get("warp_inst_per_launch"):
        return None
    name = r["kernel"].replace("void ", "").split("<")[0]
    ms = next((v["ms_per_launch"] for k, v in per_class.items() if k == name), None)
    if ms is None:
        return None
    peak = sm_count * 4 * clock_mhz * 1e6
    achieved = r["warp_inst_per_launch"] / (ms / 1e3)
    return {"bound": "alu", "kernel": name, "achieved": achieved, "peak": peak, "unit": "warp-inst/s",
            "frac": achieved / peak, "alu_pipe_pct_ncu": r.get("alu_pipe_pct"),
            "fma_pipe_pct_ncu": r.get("fma_pipe_pct"), "issue_active_pct_ncu": r.get("issue_active_pct"),
            "source": "warp instructions per launch from " + r.get("source", "profiles/")}


# ------------------------------------------------------------------ the oracle (cpu_baseline / reference arm)
def oracle_frames_per_second(workload, spec, vids, n_frames_target: int | None, seconds: float, family, seed,
                             warmup: int = 0):
    """Render output frames of batch (epoch 0, rank 0, it 0) with the oracle, one by one.

    Returns (frames, elapsed_s). Stops after n_frames_target frames, else after `seconds`.
    """
    import oracle
    import synth
    ospec = _oracle_spec(spec)
    ods = oracle.make_dataset(vids)
    metas = oracle.plan_batch(ospec, ods, len(vids), 0, 0, 0)
    W, H = workload.width, workload.height
    order = [(b, k, t) for b in range(spec.batch_size) for k, v in enumerate(spec.views) for t in range(v.clip_len)]
    frames_cache = {}

    def src(video, frame):
        key = (video, frame)
        if key not in frames_cache:
            y, uv = synth.frames(family, seed, video, frame, 1, W, H)
            frames_cache[key] = (y[0], uv[0])
        return frames_cache[key]

    # pre-generate the source frames (input generation is not the oracle's work)
    need = order if n_frames_target is None else [order[i % len(order)] for i in range(n_frames_target + warmup)]
    for b, k, t in need[: min(len(need), 4 * len(order))]:
        src(metas[b].video, metas[b].frames[k][t])
    for i in range(warmup):
        b, k, t = order[i % len(order)]
        y, uv = src(metas[b].video, metas[b].frames[k][t])
        oracle.render_frame(ospec, metas[b], k, y, uv)
    done = 0
    t0 = time.perf_counter()
    i = warmup
    while True:
        if n_frames_target is not None and done >= n_frames_target:
            break
        if n_frames_target is None and time.perf_counter() - t0 >= seconds:
            break
        b, k, t = order[i % len(order)]
        y, uv = src(metas[b].video, metas[b].frames[k][t])
        oracle.render_frame(ospec, metas[b], k, y, uv)
        done += 1
        i += 1
    return done, time.perf_counter() - t0


def _oracle_spec(spec):
    import oracle
    views = [oracle.ViewDesc(clip_len=v.clip_len, stride=v.stride, pool_offset=v.pool_offset,
                             spatial_group=v.spatial_group, geom=v.geom, scale=v.scale, ratio=v.ratio,
                             short_side=v.short_side, out_h=v.out_h, out_w=v.out_w, flip_p=v.flip_p,
                             rot_p=v.rot_p, rot_max_deg=v.rot_max_deg, blur_p=v.blur_p, sigma=v.sigma,
                             blur_ksize=v.blur_ksize, blur_truncate=v.blur_truncate, mean=v.mean, std=v.std,
                             out_dtype=v.out_dtype, subsample_of=v.subsample_of,
                             color_matrix=v.color_matrix, jitter_p=v.jitter_p, brightness=v.brightness,
                             contrast=v.contrast, saturation=v.saturation) for v in spec.views]
    return oracle.make_spec(oracle.SpecDesc(seed=spec.seed, world_size=spec.world_size,
                                            batch_size=spec.batch_size, samples_per_video=spec.samples_per_video,
                                            drop_last=spec.drop_last, shared_window=spec.shared_window, pool_epochs=spec.pool_epochs,
                                            views=views))


def max_over_ranks(values, world, device):
    """Element-wise max over ranks of a list of floats (the timed region's slowest rank)."""
    import torch
    t = torch.tensor(values, dtype=torch.float64, device=device)
    if world > 1:
        import torch.distributed as dist
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    return [float(x) for x in t.tolist()]


def gather_counters(counts, world, device):
    """All-gather per-rank integer counters and sum them (the only collective of the run)."""
    import torch
    mine = torch.tensor(counts, dtype=torch.int64, device=device)
    if world > 1:
        import torch.distributed as dist
        gathered = [torch.zeros_like(mine) for _ in range(world)]
        dist.all_gather(gathered, mine)
        return [int(x) for x in torch.stack(gathered).sum(0).tolist()], [g.tolist() for g in gathered]
    return [int(x) for x in mine.tolist()], [mine.tolist()]


def frames_per_step(spec):
    return spec.batch_size * sum(v.clip_len for v in spec.views)


def config_dict(workload, spec, n_store_videos):
    v0 = spec.views[0]
    return {"workload": workload.name, "batch_per_rank": spec.batch_size,
            "views": [{"T": v.clip_len, "stride": v.stride, "out": [v.out_h, v.out_w], "group": v.spatial_group,
                       "geom": "rrc" if v.geom == 0 else "shortside", "rot_p": v.rot_p, "blur_p": v.blur_p}
                      for v in spec.views],
            "source": [workload.width, workload.height], "store_videos_per_gpu": n_store_videos,
            "frames_per_video": workload.n_frames, "shared_window": bool(spec.shared_window),
            "out_dtype": {0: "u8", 1: "bf16", 2: "f32"}[v0.out_dtype],
            "l2": "inputs larger than L2: replicated store of %.1f GB per GPU, fresh clips every step, "
                  "per-step output > L2 for all but tiny" % (n_store_videos * workload.n_frames *
                                                              workload.frame_bytes / 1e9)}


# ------------------------------------------------------------------ reference arm
def run_reference(args):
    rank, world, local = dist_env()
    if rank != 0:
        return 0
    from paper_conf_sosp_yelllhkh25_b200 import configs
    import synth
    w = configs.get(args.config)
    spec = w.spec
    spec.world_size = 1
    vids = [(1000 + i, w.n_frames, w.width, w.height) for i in range(w.n_videos)]
    steps, warm = args.steps, args.warmup
    done, el = oracle_frames_per_second(w, spec, vids, steps, 0.0, synth.UNIFORM, 1234, warmup=warm)
    value = done / el
    line = {"impl": "reference", "metric": "output frames/s", "value": value, "unit": "frames/s",
            "n_gpus": args.gpus, "steps": steps, "warmup": warm, "ms_per_step": 1000.0 * el / max(done, 1),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u8/fp32 (oracle)",
            "data": "synthetic", "config": config_dict(w, spec, w.n_videos),
            "cpu_baseline": {"value": value, "unit": "frames/s", "cores": 1, "kind": "oracle",
                             "sample": f"one output frame per step: {done} frames of batch (epoch 0, rank 0, it 0), "
                                       f"single-threaded C oracle"},
            "e2e": {"value": value, "unit": "frames/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)
    return 0


# ------------------------------------------------------------------ our arm
def run_sand(args):
    import torch
    import torch.distributed as dist

    import synth
    import paper_conf_sosp_yelllhkh25_b200 as sand
    from paper_conf_sosp_yelllhkh25_b200 import configs

    rank, world, local = dist_env()
    if world != args.gpus:
        log(f"warning: --gpus {args.gpus} but WORLD_SIZE={world}; using WORLD_SIZE")
    # one process per GPU over NCCL; --backend gloo (tests) lets several ranks share a device
    if args.backend == "gloo":
        local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    if world > 1:
        if args.backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group("gloo")
    coll_dev = f"cuda:{local}" if args.backend == "nccl" else "cpu"
    w = configs.get(args.config)
    spec = w.spec
    spec.world_size = world
    if args.pool_epochs:
        spec.pool_epochs = args.pool_epochs
    n_videos = w.n_videos if args.videos is None else args.videos
    vids = [(1000 + i, w.n_frames, w.width, w.height) for i in range(n_videos)]
    pitch = (w.width + 63) // 64 * 64
    frame_stride = (pitch * w.height * 3 // 2 + 255) // 256 * 256
    cap = n_videos * w.n_frames * frame_stride + (64 << 20)
    t0 = time.time()
    store = sand.Store(local, cap)
    stream = torch.cuda.Stream(local)
    with torch.cuda.stream(stream):
        synth.fill_store(store, vids, synth.UNIFORM, 1234, stream.cuda_stream)
    stream.synchronize()
    log(f"[rank {rank}] store filled: {n_videos} videos, {cap / 1e9:.1f} GB in {time.time() - t0:.1f}s")
    view = sand.View(store, spec, [v[0] for v in vids])
    if args.object_budget_gb:         # f2: HBM-budgeted cache of resized frames (R#27)
        view.set_object_budget(int(args.object_budget_gb * 1e9))
    iters = view.iterations(0, rank)
    outs_a = view.alloc_outputs()
    outs_b = view.alloc_outputs()
    fps = frames_per_step(spec)

    def step_id(s):
        return s // iters, s % iters

    # the library plans epoch e+1 on its worker when epoch e's first batch is read
    view.prefetch_epoch(0, rank)

    # algorithmic bytes of the timed batches (host-side, before the warm-up so that the timed
    # region follows the warm-up directly)
    first_timed = args.warmup
    sample = sorted({step_id(first_timed + i) for i in range(0, args.steps, max(1, args.steps // 16))})
    bb = [view.batch_bytes(e, rank, it) for e, it in sample]
    alg_read = sum(b.src_bytes for b in bb) / len(bb)
    alg_write = sum(b.out_bytes for b in bb) / len(bb)

    # clock sampling starts before the warm-up so the timed region follows the warm-up steps
    # with no idle gap (an idle GPU drops to a low-power state and the first step pays for it)
    kstart = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    kend = [torch.cuda.Event(enable_timing=True) for _ in range(args.steps)]
    start = torch.cuda.Event(enable_timing=True)
    end = torch.cuda.Event(enable_timing=True)
    # no Python garbage collection from the warm-up to the end of the timed loop: a full
    # collection stalls the launching thread for milliseconds, longer than the queued GPU work
    gc.collect()
    gc.disable()
    clocks = ClockSampler(local)
    clocks.start()
    time.sleep(0.2)
    s = 0
    for _ in range(args.warmup):
        e, it = step_id(s)
        view.read_batch(e, rank, it, outs_a if s % 2 == 0 else outs_b, stream.cuda_stream)
        s += 1
    stream.synchronize()

    first_timed = s
    st0 = view.stats()
    launches0 = st0.kernel_launches
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    # the timed region holds nothing but the K read_batch calls (no per-step events between them,
    # so consecutive batches' kernels may overlap through programmatic dependent launch);
    # per-step statistics come from a separate, untimed pass below
    start.record(stream)
    for i in range(args.steps):
        e, it = step_id(s)
        if args.step_events:
            kstart[i].record(stream)
        view.read_batch(e, rank, it, outs_a if s % 2 == 0 else outs_b, stream.cuda_stream)
        if args.step_events:
            kend[i].record(stream)
        s += 1
    end.record(stream)
    torch.cuda.synchronize()
    gc.enable()
    if world > 1:
        dist.barrier()
    clk = clocks.stop()
    st1 = view.stats()
    launches = st1.kernel_launches - launches0
    host = {"read_batch_us": (st1.read_ns - st0.read_ns) / 1e3 / args.steps,
            "plan_wait_us": (st1.plan_wait_ns - st0.plan_wait_ns) / 1e3 / args.steps,
            "plans_built": int(st1.plans_built - st0.plans_built),
            "plan_cpu_ms_each": (st1.plan_cpu_ns - st0.plan_cpu_ns) / 1e6 / max(1, st1.plans_built - st0.plans_built),
            "plan_buffer_wait_ms": (st1.plan_buffer_wait_ns - st0.plan_buffer_wait_ns) / 1e6,
            "lock_wait_us": (st1.lock_wait_ns - st0.lock_wait_ns) / 1e3 / args.steps,
            "pending_waits": int(st1.pending_waits - st0.pending_waits),
            "plan_build_ms_each": ((st1.plan_build_ns - st0.plan_build_ns) / 1e6 /
                                   max(1, st1.plans_built - st0.plans_built))}
    elapsed_ms = start.elapsed_time(end)
    elapsed_ms = max_over_ranks([elapsed_ms], world, coll_dev)[0]
    ms_per_step = elapsed_ms / args.steps
    value = fps * args.steps * world / (elapsed_ms / 1000.0)

    # reuse counters of the warm-up + timed batches: the only collective (an all_gather of a few
    # integers over NCCL)
    c = store.counters()
    totals, per_rank = gather_counters([c.fetches, c.uses, c.batches], world, coll_dev)
    s_stat = s
    for i in range(args.steps):                      # per-step event timing (not the bench value)
        e, it = step_id(s_stat)
        kstart[i].record(stream)
        view.read_batch(e, rank, it, outs_a if s_stat % 2 == 0 else outs_b, stream.cuda_stream)
        kend[i].record(stream)
        s_stat += 1
    torch.cuda.synchronize()
    kraw = [a.elapsed_time(b) for a, b in zip(kstart, kend)]
    kt = sorted(kraw)
    kernel_ms = sum(kt) / args.steps
    host["kernel_ms_p10_p50_p90"] = [kt[len(kt) // 10], kt[len(kt) // 2], kt[(9 * len(kt)) // 10]]
    slow = [(i, round(x, 3)) for i, x in enumerate(kraw) if x > 2 * kt[len(kt) // 2]]
    host["slow_steps"] = {"n": len(slow), "ms_total": round(sum(x for _, x in slow), 3),
                          "first": [(first_timed + args.steps + i, x) for i, x in slow[:8]], "iters_per_epoch": iters,
                          "note": "per-step events from an untimed pass over the next K batches"}

    # per-kernel roofline: each item class is its own kernel; time each class with
    # CUDA events recorded by the library around its launch, on the stream it runs on, over a
    # separate pass of the same batches (so the timed loop above carries no timing events)
    cls_names = CLASS_KERNELS.get(args.config, DEFAULT_CLASS_KERNELS)
    view.set_timing(True)
    n_cls_steps = min(args.steps, 200)
    s_cls = first_timed
    for _ in range(n_cls_steps):
        e, it = step_id(s_cls)
        view.read_batch(e, rank, it, outs_a if s_cls % 2 == 0 else outs_b, stream.cuda_stream)
        s_cls += 1
    cls_ms, cls_n = view.class_times()
    view.set_timing(False)
    cls_bytes = [[0.0, 0.0] for _ in range(3)]
    for e, it in sample:
        for c in range(3):
            b = view.batch_bytes_class(e, rank, it, c)
            cls_bytes[c][0] += b.src_bytes / len(sample)
            cls_bytes[c][1] += b.out_bytes / len(sample)
    per_class = {}
    for c in range(3):
        if cls_n[c]:
            ms_each = cls_ms[c] / cls_n[c]
            per_class[cls_names[c]] = {"ms_per_launch": ms_each, "launches": int(cls_n[c]),
                                       "alg_bytes_per_launch": {"read": cls_bytes[c][0], "write": cls_bytes[c][1]},
                                       "achieved_gbs": (cls_bytes[c][0] + cls_bytes[c][1]) / (ms_each / 1e3) / 1e9}
    dom = max(per_class, key=lambda k: per_class[k]["ms_per_launch"] * per_class[k]["launches"]) if per_class else None



    # ---- e2e through the C-ABI with HOST buffers
    e2e = None
    if not args.no_e2e:
        e2e = run_e2e(args, w, spec, view, store, stream, rank, iters, s, world, coll_dev)

    peak, peak_src = measured_peaks()
    step_achieved = (alg_read + alg_write) / (kernel_ms / 1000.0) / 1e9
    achieved = per_class[dom]["achieved_gbs"] if dom else step_achieved
    line = {
        "metric": "output frames/s", "value": value, "unit": "frames/s", "n_gpus": world, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": ms_per_step, "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": {0: "u8", 1: "bf16", 2: "f32"}[spec.views[0].out_dtype],
        "data": "synthetic (seeded NV12, uniform family)", "config": config_dict(w, spec, n_videos),
        "batches_per_s": value / fps,
        "per_gpu_frames_per_s": value / world,
        "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s", "frac": achieved / peak,
                     "traffic": ncu_traffic(args.config), "kernel": dom,
                     "alg_bytes_per_launch": (per_class[dom]["alg_bytes_per_launch"] if dom else
                                              {"read": alg_read, "write": alg_write}),
                     "ms_per_launch": per_class[dom]["ms_per_launch"] if dom else kernel_ms,
                     "per_kernel": per_class,
                     "step": {"achieved": step_achieved, "frac": step_achieved / peak, "kernel_ms_per_step": kernel_ms,
                              "alg_bytes": {"read": alg_read, "write": alg_write}},
                     "peak_source": peak_src, "frac_of_8tbs_spec": achieved / 8000.0},
        "roofline_alu": alu_roofline(args.config, per_class, torch.cuda.get_device_properties(local).multi_processor_count,
                                     float(clk.get("sm_max_mhz") or 1965.0)),
        "gpu_launches": int(launches),
        "object_cache": (None if not args.object_budget_gb else
                         {k: int(getattr(view.object_stats(), k)) for k in
                          ("hits", "fills", "misses", "evictions", "objects", "bytes_used", "bytes_budget",
                           "decide_ns", "stage_ns", "launch_ns")}),
        "host": host,
        "clocks": clk,
        "reuse": {"fetches": totals[0], "uses": totals[1], "batches": totals[2], "per_rank": per_rank},
        "collectives": {"backend": args.backend if world > 1 else None,
                        "timing": "max over ranks of CUDA-event times", "counters": "all_gather"},
    }
    if e2e is not None:
        line["e2e"] = e2e
    if rank == 0 and not args.no_cpu:
        line["cpu_baseline"] = cpu_baseline(w, spec, vids, args)
    if rank == 0:
        print(json.dumps(line), flush=True)
    view.close()
    store.close()
    if world > 1:
        dist.destroy_process_group()
    return 0


def run_e2e(args, w, spec, view, store, stream, rank, iters, s0, world, coll_dev):
    """Same metric end to end through the public API: every step copies its input frames
    from pinned host memory into the store (one sand_store_put_frame_batch: one H2D copy of
    the packed frames + one scatter kernel), reads the batch, and copies the batch back to
    pinned host memory (D2H). The D2H of step i runs on a copy stream while step i + 1's
    H2D and kernels run (double-buffered outputs), so the two PCIe directions overlap; the
    timed region ends when the last D2H has landed."""
    import torch
    import synth
    n = args.e2e_steps
    steps = [((s0 + i) // iters, (s0 + i) % iters) for i in range(n)]
    W, H = w.width, w.height
    fb = W * H * 3 // 2
    # stage each step's unique source frames in pinned host memory (outside the timed region)
    staged = []
    scratch = torch.empty(fb, dtype=torch.uint8, device=f"cuda:{torch.cuda.current_device()}")
    for e, it in steps:
        keys = sorted({(m.video, m.frames[k][t]) for m in view.get_meta(e, rank, it)
                       for k, v in enumerate(spec.views) for t in range(v.clip_len)})
        host = torch.empty((len(keys), fb), dtype=torch.uint8, pin_memory=True)
        for i, (vid, f) in enumerate(keys):
            synth.fill_device(synth.UNIFORM, 1234, vid, f, 1, W, H, scratch.data_ptr(), W,
                              scratch.data_ptr() + W * H, W, 0, 0)
            host[i].copy_(scratch)
        staged.append((keys, host))
    outs2 = [view.alloc_outputs(), view.alloc_outputs()]
    host_out = [[torch.empty(o.shape, dtype=o.dtype, pin_memory=True) for o in outs] for outs in outs2]
    h2d = sum(len(k) * fb for k, _ in staged) / n
    d2h = sum(o.numel() * o.element_size() for o in outs2[0])
    copy_stream = torch.cuda.Stream()
    ready = [torch.cuda.Event(), torch.cuda.Event()]
    drained = [torch.cuda.Event(), torch.cuda.Event()]
    # untimed warm-up of the batch-put path (staging buffers are allocated on first use)
    keys0, host0 = staged[0]
    store.put_frame_batch([k[0] for k in keys0], [k[1] for k in keys0], host0.data_ptr(), fb, W, W * H, False,
                          stream.cuda_stream)
    torch.cuda.synchronize()
    start = torch.cuda.Event(enable_timing=True)
    end = torch.cuda.Event(enable_timing=True)
    start.record(stream)
    for i, ((e, it), (keys, host)) in enumerate(zip(steps, staged)):
        j = i % 2
        if i >= 2:
            stream.wait_event(drained[j])      # buffer j's previous D2H has landed
        store.put_frame_batch([k[0] for k in keys], [k[1] for k in keys], host.data_ptr(), fb, W, W * H, False,
                              stream.cuda_stream)
        view.read_batch(e, rank, it, outs2[j], stream.cuda_stream)
        ready[j].record(stream)
        copy_stream.wait_event(ready[j])
        with torch.cuda.stream(copy_stream):
            for ho, o in zip(host_out[j], outs2[j]):
                ho.copy_(o, non_blocking=True)
        drained[j].record(copy_stream)
    stream.wait_stream(copy_stream)
    end.record(stream)
    torch.cuda.synchronize()
    ms = max_over_ranks([start.elapsed_time(end)], world, coll_dev)[0]
    return {"value": frames_per_step(spec) * n * world / (ms / 1000.0), "unit": "frames/s",
            "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h), "steps": n,
            "ms_per_step": ms / n, "api": "sand_store_put_frame_batch + sand_view_read_batch, D2H overlapped"}


def cpu_model() -> str:
    try:
        out = subprocess.run(["lscpu"], capture_output=True, text=True, timeout=10).stdout
        for ln in out.splitlines():
            if ln.startswith("Model name:"):
                return ln.split(":", 1)[1].strip()
    except (OSError, subprocess.SubprocessError):
        pass
    return "unknown"


def _oracle_worker(config, cpu, index, procs, seconds, q):
    """One pinned oracle process: renders output frames index, index + procs, ... of the
    workload's batches (disjoint across processes) for `seconds` (the box-level
    CPU rate, P = os.cpu_count() pinned processes over disjoint clips)."""
    try:
        os.sched_setaffinity(0, {cpu})
    except (AttributeError, OSError):
        pass
    import oracle
    import synth
    from paper_conf_sosp_yelllhkh25_b200 import configs
    w = configs.get(config)
    spec = w.spec
    spec.world_size = 1
    vids = [(1000 + i, w.n_frames, w.width, w.height) for i in range(w.n_videos)]
    ospec = _oracle_spec(spec)
    ods = oracle.make_dataset(vids)
    order = []
    it = 0
    while len(order) < 4 * procs and it < oracle.iterations(ospec, len(vids)):
        metas = oracle.plan_batch(ospec, ods, len(vids), 0, 0, it)
        order += [(metas[b], k) + (metas[b].frames[k][t],) for b in range(spec.batch_size)
                  for k, v in enumerate(spec.views) for t in range(v.clip_len)]
        it += 1
    mine = order[index::procs][:64]
    src = {}
    for m, k, f in mine:           # source frames generated before the clock starts
        if (m.video, f) not in src:
            y, uv = synth.frames(synth.UNIFORM, 1234, m.video, f, 1, w.width, w.height)
            src[(m.video, f)] = (y[0], uv[0])
    done, t0 = 0, time.perf_counter()
    while time.perf_counter() - t0 < seconds:
        m, k, f = mine[done % len(mine)]
        y, uv = src[(m.video, f)]
        oracle.render_frame(ospec, m, k, y, uv)
        done += 1
    q.put((done, time.perf_counter() - t0))


def cpu_baseline(w, spec, vids, args):
    """The oracle as it stands on the box's host cores: one pinned process per core over
    disjoint output frames (box rate), the single-core rate, the CPU model and the paper's
    12-cores-per-GPU provisioning as context."""
    import multiprocessing as mp
    import synth
    done1, el1 = oracle_frames_per_second(w, spec, vids, None, min(args.cpu_seconds, 6.0), synth.UNIFORM, 1234,
                                          warmup=1)
    try:
        cpus = sorted(os.sched_getaffinity(0))
    except AttributeError:
        cpus = list(range(os.cpu_count() or 1))
    procs = len(cpus)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_oracle_worker, args=(args.config, cpus[i], i, procs, args.cpu_seconds, q))
          for i in range(procs)]
    for p in ps:
        p.start()
    res = [q.get(timeout=600) for _ in ps]
    for p in ps:
        p.join()
    box = sum(d / e for d, e in res)
    return {"value": box, "unit": "frames/s", "cores": procs, "kind": "oracle",
            "cpu_model": cpu_model(),
            "sample": f"{procs} pinned processes (one per host core), each rendering disjoint output frames of the "
                      f"workload's first batches one by one with the single-threaded C oracle for "
                      f"{args.cpu_seconds:.0f}s (source-frame generation excluded); box rate = sum of per-process rates",
            "single_core": {"value": done1 / el1, "frames": done1, "seconds": round(el1, 2)},
            "per_12_cores": box * 12.0 / procs,
            "per_12_cores_note": "the paper provisions 12 CPU cores per GPU (P:L120, P:L414): box rate x 12 / cores"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=None)
    ap.add_argument("--warmup", type=int, default=20)
    ap.add_argument("--config", default="k400", choices=["tiny", "k400", "slowfast", "twoview", "ray", "slowfast_hd"])
    ap.add_argument("--impl", default="sand", choices=["sand", "reference"])
    ap.add_argument("--videos", type=int, default=None, help="override the store size (videos per GPU)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=16)
    ap.add_argument("--pool-epochs", type=int, default=0, help="k-epoch shared frame pool (f1, R#25)")
    ap.add_argument("--object-budget-gb", type=float, default=0.0, help="HBM object cache (f2, R#27)")
    ap.add_argument("--step-events", action="store_true",
                    help="diagnostics: record per-step CUDA events inside the timed loop")
    ap.add_argument("--backend", default="nccl", choices=["nccl", "gloo"],
                    help="process-group backend (gloo: test mode, ranks may share one GPU)")
    ap.add_argument("--cpu-seconds", type=float, default=10.0)
    args = ap.parse_args()
    if args.steps is None:
        args.steps = DEFAULT_STEPS[args.config] if args.impl == "sand" else 200
    args.warmup = max(args.warmup, 3)
    if args.impl == "reference":
        return run_reference(args)
    return run_sand(args)


if __name__ == "__main__":
    sys.exit(main())
