#!/usr/bin/env python
"""§8(f) f1 measurement (Fig. 19 analogue): how often each selected frame is
selected over ten epochs, per-epoch pools (k = 1) vs k-epoch pools, with the oracle planner on
synthetic 300-frame videos (the product planner is bit-identical: tests/test_planner_host.py).

    python tools/pool_reuse.py
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))
import oracle  # noqa: E402
from paper_conf_sosp_yelllhkh25_b200 import configs  # noqa: E402
from helpers import to_oracle  # noqa: E402


def counts(name, k, n_videos=128, epochs=10):
    w = configs.get(name)
    w.spec.pool_epochs = k
    ospec = to_oracle(w.spec)
    vids = [(1000 + i, 300, w.width, w.height) for i in range(n_videos)]
    ods = oracle.make_dataset(vids)
    c = {}
    for e in range(epochs):
        for clip in range(n_videos * w.spec.samples_per_video):
            m = oracle.ClipMeta()
            oracle.lib().oracle_plan_clip(oracle.ctypes.byref(ospec), ods, e, clip, oracle.ctypes.byref(m))
            frames = {m.frames[v][t] for v, vd in enumerate(w.spec.views) for t in range(vd.clip_len)}
            for f in frames:
                c[(m.video, f)] = c.get((m.video, f), 0) + 1
    return np.array(list(c.values()))


if __name__ == "__main__":
    for name in ("k400", "slowfast", "twoview"):
        for k in (1, 5, 10):
            c = counts(name, k)
            print(f"{name:9s} k={k:2d}: frames selected {len(c):6d}, chosen >= 4 times {100 * np.mean(c >= 4):5.1f} %,"
                  f" mean selections {c.mean():.2f}")
