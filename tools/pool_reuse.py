#!/usr/bin/env python
"""§8(f) f1 measurement: the Fig. 19 / Fig. 16 analogue (§7.4) with the product's
host planner (sand_plan_clip, the planner read_batch uses) on synthetic 300-frame videos.

Fig. 19 is measured on the paper's TWO-TASK workload (SlowFast and MAE trained together):
"Without SAND, only 10.6 % of frames are chosen four or more times [over ten epochs]; with SAND
the share climbs to 60.1 %". Here:
  * without SAND: the two tasks plan independently (two view groups with their own seeds, a
    fresh frame pool per task and epoch, k = 1);
  * with SAND: one view group holding both tasks (shared GCD frame pool across tasks)
    and the k-epoch pool, k in {1, 5, 10}.
It reports the share of selected frames chosen >= 4 times over ten epochs, and the distinct
frames decoded per epoch (Fig. 16's decode operations, "50.3 % reduction").

    python tools/pool_reuse.py [n_videos]
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import paper_conf_sosp_yelllhkh25_b200 as sand  # noqa: E402
from paper_conf_sosp_yelllhkh25_b200 import configs  # noqa: E402

V = configs.ViewSpec


def slowfast_view(group):
    # SlowFast's fast pathway (32 frames, stride 2; the slow pathway is a subset of it)
    return V(clip_len=32, stride=2, spatial_group=group, geom=configs.GEOM_SHORTSIDE_CROP, short_side=256)


def mae_view(group):
    # VideoMAE pre-training on Kinetics: 16 frames at sampling rate 4
    return V(clip_len=16, stride=4, spatial_group=group)


def selections(specs, n_videos, epochs):
    """(video, frame) -> times selected over `epochs`, summed over the given view groups, and the
    mean number of distinct frames decoded per epoch."""
    vids = [(1000 + i, 300, 340, 256) for i in range(n_videos)]
    c, decoded = {}, []
    for e in range(epochs):
        epoch_frames = set()
        for spec in specs:
            for clip in range(n_videos * spec.samples_per_video):
                m = sand.plan_clip(spec, vids, e, clip)
                for k, v in enumerate(spec.views):     # one selection per task (view) that picked the frame
                    for f in {m.frames[k][t] for t in range(v.clip_len)}:
                        c[(m.video, f)] = c.get((m.video, f), 0) + 1
                        epoch_frames.add((m.video, f))
        decoded.append(len(epoch_frames))
    return np.array(list(c.values())), float(np.mean(decoded))


def report(label, cnt, decoded):
    line = (f"{label:44s} frames selected {len(cnt):6d}  chosen >= 4 times {100 * np.mean(cnt >= 4):5.1f} %  "
            f"decoded per epoch {decoded:8.0f}")
    print(line)
    return line


if __name__ == "__main__":
    n = int(sys.argv[1]) if len(sys.argv) > 1 else 128
    epochs = 10
    lines = [f"# Fig. 19 / Fig. 16 analogue: SlowFast + MAE on {n} synthetic 300-frame videos, {epochs} epochs",
             "# (P:L494-498: without SAND 10.6 % of frames chosen >= 4 times, with SAND 60.1 %; decoding -50.3 %)"]
    sep = [configs.Spec(seed=1, views=[slowfast_view(0)]), configs.Spec(seed=2, views=[mae_view(0)])]
    cnt, dec0 = selections(sep, n, epochs)
    lines.append(report("without sharing (two tasks, own pools, k=1)", cnt, dec0))
    for k in (1, 5, 10):
        shared = [configs.Spec(seed=1, pool_epochs=k, views=[slowfast_view(0), mae_view(1)])]
        cnt, dec = selections(shared, n, epochs)
        lines.append(report(f"shared pool across tasks, k={k}", cnt, dec) +
                     f"  decode reduction {100 * (1 - dec / dec0):5.1f} %")
    for name in ("k400", "slowfast"):
        for k in (1, 10):
            w = configs.get(name)
            w.spec.pool_epochs = k
            cnt, dec = selections([w.spec], n, epochs)
            lines.append(report(f"single task {name}, k={k}", cnt, dec))
    out = os.path.join(ROOT, "profiles", "r02_pool_reuse.txt")
    with open(out, "w") as f:
        f.write("\n".join(lines) + "\n")
    print("wrote", out)
