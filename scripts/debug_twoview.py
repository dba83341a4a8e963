"""Diagnose stencil-path mismatches: which (clip, view, t, channel, pixel) differ, with meta."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np, torch
import oracle, synth
import paper_conf_sosp_yelllhkh25_b200 as sand
from paper_conf_sosp_yelllhkh25_b200 import configs
from helpers import to_oracle, videos_of, oracle_render, out_numpy

w = configs.twoview()
w.spec.batch_size = 8
for v in w.spec.views:
    v.out_dtype = configs.U8
vids = videos_of(w, 24)
store = sand.Store(0, 24 * 300 * 147456 + (1 << 20))
synth.fill_store(store, vids, synth.UNIFORM, 1234)
view = sand.View(store, w.spec, [v[0] for v in vids])
ospec = to_oracle(w.spec)
ods = oracle.make_dataset(vids)
outs = view.alloc_outputs()
view.read_batch(1, 0, 0, outs)
torch.cuda.synchronize()
metas = oracle.plan_batch(ospec, ods, 24, 1, 0, 0)
for b in range(8):
    m = metas[b]
    for k in range(2):
        for t in (0, 7):
            ref = oracle_render(ospec, m, k, t, synth.UNIFORM, 1234, 340, 256).astype(np.int32)
            got = out_numpy(outs[k][b, :, t]).astype(np.int32)
            d = np.abs(got - ref)
            q = k
            tag = f"b={b} k={k} t={t} rot={m.rot_on[q]} th={m.theta[q]:.3f} blur={m.blur_on[q]} r={m.blur_r[q]} flip={m.flip[q]}"
            if d.max() > 0:
                idx = np.argwhere(d > 0)
                print(tag, "MISMATCH n=%d max=%d" % (len(idx), d.max()), "first", idx[:5].tolist(),
                      "rows", sorted(set(idx[:, 1].tolist()))[:20])
            else:
                print(tag, "ok")
