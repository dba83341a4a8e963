"""Pins of the f2 object-cache oracle (oracle/object_cache.py; R#27) by closed forms.

With pool_offset 0 (SlowFast pathways) every epoch of a k-epoch chunk selects the same frames
for a clip (R#25), so with room for every object: k = 1 never fills (no later use: Alg. 1 keeps
the leaves), and k = 2 fills every (video, frame) once in the chunk's first epoch and hits all of
them in its second; a zero budget misses everything.
"""
import oracle
from oracle import object_cache
from oracle import SpecDesc, ViewDesc, GEOM_SHORTSIDE_CROP


def _spec(k):
    v = dict(pool_offset=0, geom=GEOM_SHORTSIDE_CROP, short_side=48, out_h=32, out_w=32)
    return oracle.make_spec(SpecDesc(seed=5, batch_size=2, pool_epochs=k, views=[
        ViewDesc(clip_len=8, stride=2, **v), ViewDesc(clip_len=2, stride=8, **v)]))


def test_closed_forms():
    ds = oracle.make_dataset([(10 + i, 60, 96, 64) for i in range(4)])
    reads = [(e, it) for e in range(2) for it in range(2)]
    per_epoch = 4 * 8                       # 4 clips x 8 distinct fast frames (slow subset)
    s1 = object_cache.simulate(_spec(1), ds, 4, 10**9, reads)[-1]
    assert (s1["fills"], s1["hits"], s1["misses"]) == (0, 0, 2 * per_epoch)
    s2 = object_cache.simulate(_spec(2), ds, 4, 10**9, reads)
    assert (s2[1]["fills"], s2[1]["hits"]) == (per_epoch, 0)           # after epoch 0
    assert (s2[-1]["fills"], s2[-1]["hits"], s2[-1]["misses"]) == (per_epoch, per_epoch, 0)
    s0 = object_cache.simulate(_spec(2), ds, 4, 0, reads)[-1]
    assert (s0["fills"], s0["hits"], s0["misses"]) == (0, 0, 2 * per_epoch)


def test_eviction_keeps_budget_and_prefers_unneeded_objects():
    ds = oracle.make_dataset([(10 + i, 60, 96, 64) for i in range(4)])
    spec = _spec(3)
    objbytes = 3 * 72 * 48                                     # W' = 96 * 48 / 64 = 72, H' = 48
    budget = 10 * objbytes + 16
    reads = [(e, it) for e in range(6) for it in range(2)]
    out = object_cache.simulate(spec, ds, 4, budget, reads)
    assert all(o["objects"] * objbytes * 4 <= budget * 3 for o in out)    # 75 % after every batch
    assert out[-1]["evictions"] > 0 and out[-1]["hits"] > 0
