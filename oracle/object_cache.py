"""Oracle of the f2 object-cache policy (TEST INFRASTRUCTURE ONLY; R#27).

Restates, step by step, the decisions read_batch takes for the HBM-budgeted object cache
(§5.3 Alg. 1, §6), driven by the C oracle's planner:

  * eligible items: (clip slot b, frame f, group q) whose group leader view is a short-side crop
    without rotation/blur, visited per batch in (b, f, q) order;
  * later(item) = number of later epochs of the current k-epoch chunk in which clip b's plan
    selects frame f for group q (a chunk's pool is decoded once and reused);
  * HIT if (video, f) is cached; else FILL if later >= 1 (Alg. 1: caching the parent saves the
    space of its >= 2 leaves) and a slot is free, evicting one object first when none is;
    else MISS;
  * eviction (§6): among objects not touched by the current batch, first those not needed again
    in the current chunk (least recently used first), then the one with the latest next use;
    after each batch, evict while more than 75 % of the budget is in use.
Slots: budget // objbytes with objbytes = 3 W' H' + 16 rounded up to 256.
"""
from __future__ import annotations

import oracle

GEOM_SHORTSIDE_CROP = oracle.GEOM_SHORTSIDE_CROP


def _eligible_groups(spec):
    lead = {}
    for k in range(spec.n_views):
        q = spec.views[k].spatial_group
        lead.setdefault(q, k)
    return {q for q, k in lead.items() if spec.views[k].geom == GEOM_SHORTSIDE_CROP
            and spec.views[k].rot_p <= 0 and spec.views[k].blur_p <= 0}


def simulate(spec, dataset, n_videos, budget, reads):
    """reads: list of (epoch, iteration) for rank 0 in read order. Returns per-read dicts of
    hits, fills, misses, evictions (cumulative) and cached objects."""
    kch = max(1, spec.pool_epochs)
    elig = _eligible_groups(spec)
    objs = {}                     # (video, frame) -> dict(slot, remaining, chunk, next, last)
    free, n_slots, objbytes, size = [], 0, 0, None
    st = {"hits": 0, "fills": 0, "misses": 0, "evictions": 0}
    out = []
    seq = 0

    def evict_to_threshold(epoch, chunk, protect):
        cands = []
        for key, o in objs.items():
            if protect and o["last"] == seq:
                continue
            needed = o["remaining"] > 0 and o["chunk"] == chunk and o["next"] is not None and o["next"] >= epoch
            cands.append(((1, -o["next"], o["last"]) if needed else (0, o["last"], 0), key))
        for _, key in sorted(cands):
            if len(objs) * objbytes * 4 <= budget * 3:
                break
            free.append(objs.pop(key)["slot"])
            st["evictions"] += 1

    for epoch, it in reads:
        seq += 1
        chunk = epoch // kch
        metas = oracle.plan_batch(spec, dataset, n_videos, epoch, 0, it)
        items = []
        for b, m in enumerate(metas):
            for q in sorted(elig):
                frames = sorted({m.frames[k][t] for k in range(spec.n_views) if spec.views[k].spatial_group == q
                                 for t in range(spec.views[k].clip_len)})
                later = {}
                for e2 in range(epoch + 1, (chunk + 1) * kch):
                    m2 = oracle.ClipMeta()
                    oracle.lib().oracle_plan_clip(oracle.ctypes.byref(spec), dataset, e2, m.clip, oracle.ctypes.byref(m2))
                    sel = {m2.frames[k][t] for k in range(spec.n_views) if spec.views[k].spatial_group == q
                           for t in range(spec.views[k].clip_len)}
                    for f in sel:
                        later.setdefault(f, []).append(e2)
                for f in frames:
                    items.append((b, f, q, m.video, tuple(m.box[q]), later.get(f, [])))
        for b, f, q, video, box, lat in sorted(items):
            if size is None:
                size = (box[2], box[3])
                objbytes = 3 * box[2] * box[3]
                n_slots = min((budget - 16) // objbytes if budget > 16 else 0, 65535)
                free = list(range(n_slots))[::-1]
            if (box[2], box[3]) != size:
                st["misses"] += 0            # other size classes bypass the cache (not counted)
                continue
            key = (video, f)
            cached = key in objs
            if not cached and len(lat) >= 1:
                if not free:
                    evict_to_threshold(epoch, chunk, True)
                if free:
                    objs[key] = {"slot": free.pop()}
                    cached = True
                    st["fills"] += 1
            elif cached:
                st["hits"] += 1
            if not cached:
                st["misses"] += 1
                continue
            o = objs[key]
            o.update(remaining=len(lat), chunk=chunk, next=(lat[0] if lat else None), last=seq)
        evict_to_threshold(epoch, chunk, False)
        out.append(dict(st, objects=len(objs)))
    return out
