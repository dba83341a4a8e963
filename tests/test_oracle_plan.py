"""Pins for the oracle's temporal sampling (O4) and spatial draws (O5).

O4 (shared frame pool) and the shared window are the paper's
own coordination mechanisms: they are pinned by closed forms on tiny cases,
containment and uniformity invariants ("parity unpinned beyond invariants",
DESIGN.md §5). The RRC box is pinned EXACTLY to torchvision's own
RandomResizedCrop.get_params run on the same uniforms (its RNG calls are
redirected to the oracle's Philox draws), and in distribution to torchvision's
unmodified sampler. The blur radius is pinned to scipy's truncate rule.
"""
import ctypes
import math

import numpy as np
import pytest
import scipy.ndimage
import scipy.stats
import torch

import oracle
from oracle import ViewDesc, SpecDesc

SEED = 20251013


def _spec(views, **kw):
    return oracle.make_spec(SpecDesc(seed=kw.pop("seed", SEED), views=views, **kw))


def _temporal(spec, epoch, clip, F):
    m = oracle.ClipMeta()
    oracle.lib().oracle_temporal(ctypes.byref(spec), epoch, clip, F, ctypes.byref(m))
    return m


# ---------------------------------------------------------------- O4 temporal

def test_tiny_temporal_closed_form():
    # tiny config: F=16, T=8, s=2 -> pool P=15 frames -> start in {0,1}, idx = start + 2t
    spec = _spec([ViewDesc(clip_len=8, stride=2, out_h=32, out_w=32)])
    starts = set()
    for e in range(200):
        m = _temporal(spec, e, 0, 16)
        s = m.pool_start
        starts.add(s)
        assert list(m.frames[0][:8]) == [s + 2 * t for t in range(8)]
    assert starts == {0, 1}


def test_slowfast_pool_slow_is_subset_of_fast():
    # g = gcd(2, 8) = 2; L = 32 grid points; fixed offsets 0 -> slow[j] == fast[4j]
    spec = _spec([ViewDesc(clip_len=32, stride=2, pool_offset=0, spatial_group=0),
                  ViewDesc(clip_len=8, stride=8, pool_offset=0, spatial_group=0)])
    for c in range(50):
        m = _temporal(spec, 3, c, 300)
        fast = list(m.frames[0][:32])
        slow = list(m.frames[1][:8])
        assert slow == [fast[4 * j] for j in range(8)]
        assert fast == [m.pool_start + 2 * t for t in range(32)]
        assert 0 <= m.pool_start <= 300 - 63


def test_random_offsets_stay_on_grid_inside_pool():
    spec = _spec([ViewDesc(clip_len=16, stride=4), ViewDesc(clip_len=4, stride=8, spatial_group=1),
                  ViewDesc(clip_len=8, stride=6, spatial_group=2)])
    # g = gcd(4, 8, 6) = 2; spans 31, 13, 22 grid points; L = 31; P = 61 frames
    offsets = set()
    for c in range(300):
        m = _temporal(spec, 0, c, 300)
        s = m.pool_start
        for k, (T, st) in enumerate([(16, 4), (4, 8), (8, 6)]):
            idx = list(m.frames[k][:T])
            assert all((i - s) % 2 == 0 for i in idx)                 # on the gcd grid
            assert all(s <= i <= s + 60 for i in idx)                 # inside the pool
            assert all(b - a == st for a, b in zip(idx, idx[1:]))     # the view's own stride
            offsets.add((k, (idx[0] - s) // 2))
    assert {o for k, o in offsets if k == 0} == {0}                  # the longest view spans the pool
    assert {o for k, o in offsets if k == 1} == set(range(0, 31 - 13 + 1))
    assert {o for k, o in offsets if k == 2} == set(range(0, 31 - 22 + 1))


def test_short_video_clamps_to_last_frame():
    spec = _spec([ViewDesc(clip_len=16, stride=4)])
    m = _temporal(spec, 0, 0, 10)
    assert m.pool_start == 0
    assert list(m.frames[0][:16]) == [min(4 * t, 9) for t in range(16)]


def test_clip_start_uniform():
    spec = _spec([ViewDesc(clip_len=16, stride=4)])
    F, P = 100, 61
    counts = np.zeros(F - P + 1)
    for c in range(8000):
        counts[_temporal(spec, 1, c, F).pool_start] += 1
    assert scipy.stats.chisquare(counts).pvalue > 1e-5


# ---------------------------------------------------------------- O5 spatial: RRC vs torchvision

class _FakeUniform:
    def __init__(self, feed):
        self.feed = feed

    def uniform_(self, a, b):
        u = self.feed.u01()
        a, b = float(a), float(b)
        return torch.tensor([a + (b - a) * u], dtype=torch.float64)


class _Feed:
    """Replays the oracle's Philox draws into torchvision's get_params."""

    def __init__(self, seed, epoch, clip, group):
        self.seed, self.epoch, self.clip, self.group = seed, epoch, clip, group
        self.attempt = 0
        self.k = 0
        self.x = None

    def _draw(self):
        c1 = (3 << 24) | (self.group << 16)
        return oracle.philox([self.attempt, c1, self.clip, self.epoch & 0xFFFFFFFF],
                             [self.seed & 0xFFFFFFFF, self.seed >> 32])

    def u01(self):
        if self.k == 0:
            self.x = self._draw()
        v = self.x[self.k] / 2**32
        self.k += 1
        return v

    def randint(self, lo, hi, size=None):
        # get_params draws i (rows) from x[2] then j (cols) from x[3]
        v = oracle.bounded(self.x[self.k], hi - lo) + lo
        self.k += 1
        if self.k == 4:
            self.k = 0
            self.attempt += 1
        return torch.tensor([v])

    def end_attempt(self):
        # a rejected attempt consumed x[0], x[1] only
        self.k = 0
        self.attempt += 1


def _torchvision_box(monkeypatch, W, H, scale, ratio, seed, epoch, clip, group):
    import torchvision.transforms.transforms as tvt
    feed = _Feed(seed, epoch, clip, group)
    real = torch

    class FakeTorch:
        def __getattr__(self, name):
            return getattr(real, name)

        @staticmethod
        def tensor(x, **kw):
            return real.tensor(x, dtype=real.float64)

        @staticmethod
        def empty(*a, **kw):
            if feed.k == 2:          # previous attempt was rejected after its two uniforms
                feed.end_attempt()
            return _FakeUniform(feed)

        @staticmethod
        def randint(lo, hi, size=None):
            return feed.randint(lo, hi, size)

    monkeypatch.setattr(tvt, "torch", FakeTorch())
    img = real.zeros(3, H, W)
    i, j, h, w = tvt.RandomResizedCrop.get_params(img, list(scale), list(ratio))
    monkeypatch.undo()
    return [j, i, w, h]


@pytest.mark.parametrize("W,H,scale,ratio", [
    (340, 256, (0.08, 1.0), (3 / 4, 4 / 3)),
    (1920, 1080, (0.35, 1.0), (3 / 4, 4 / 3)),
    (64, 64, (0.08, 1.0), (3 / 4, 4 / 3)),
    (340, 64, (0.9, 1.0), (3.0, 4.0)),          # attempts usually fail -> central fallback
    (64, 340, (0.9, 1.0), (0.2, 0.25)),         # fallback with in_ratio < min(ratio)
    (100, 20, (0.95, 1.0), (1.0, 1.2)),         # fallback with in_ratio > max(ratio)
])
def test_rrc_box_equals_torchvision_get_params(monkeypatch, W, H, scale, ratio):
    v = oracle.make_spec(SpecDesc(views=[ViewDesc(scale=scale, ratio=ratio)])).views[0]
    box = (ctypes.c_int32 * 4)()
    for clip in range(300):
        for group in (0, 3):
            oracle.lib().oracle_rrc_box(ctypes.byref(v), SEED, 7, clip, group, W, H, box)
            expect = _torchvision_box(monkeypatch, W, H, scale, ratio, SEED, 7, clip, group)
            assert list(box) == expect, (clip, group)


def test_rrc_distribution_matches_torchvision_sampler():
    import torchvision.transforms as T
    W, H = 340, 256
    v = oracle.make_spec(SpecDesc(views=[ViewDesc()])).views[0]
    box = (ctypes.c_int32 * 4)()
    ours = {"area": [], "x": [], "ratio": []}
    for clip in range(6000):
        oracle.lib().oracle_rrc_box(ctypes.byref(v), SEED, 0, clip, 0, W, H, box)
        ours["area"].append(box[2] * box[3])
        ours["x"].append(box[0] / max(1, W - box[2]) if W > box[2] else 0.5)
        ours["ratio"].append(box[2] / box[3])
    torch.manual_seed(0)
    img = torch.zeros(3, H, W)
    ref = {"area": [], "x": [], "ratio": []}
    for _ in range(6000):
        i, j, h, w = T.RandomResizedCrop.get_params(img, [0.08, 1.0], [3 / 4, 4 / 3])
        ref["area"].append(w * h)
        ref["x"].append(j / max(1, W - w) if W > w else 0.5)
        ref["ratio"].append(w / h)
    for k in ours:
        assert scipy.stats.ks_2samp(ours[k], ref[k]).pvalue > 1e-4, k


# ---------------------------------------------------------------- short side, window, gates

def test_shortside_box_range_and_uniformity():
    v = oracle.make_spec(SpecDesc(views=[ViewDesc(geom=oracle.GEOM_SHORTSIDE_CROP, short_side=256,
                                                  out_h=224, out_w=224)])).views[0]
    box = (ctypes.c_int32 * 4)()
    xs, ys = [], []
    for clip in range(4000):
        oracle.lib().oracle_shortside_box(ctypes.byref(v), SEED, 0, clip, 0, 1280, 720, box)
        Wp, Hp = box[2], box[3]
        assert Hp == 256 and Wp == 1280 * 256 // 720      # short side -> S, long side floored
        assert 0 <= box[0] <= Wp - 224 and 0 <= box[1] <= Hp - 224
        xs.append(box[0])
        ys.append(box[1])
    assert min(xs) == 0 and max(xs) == 455 - 224           # inclusive offset range
    assert scipy.stats.kstest((np.array(xs) + 0.5) / 232, "uniform").pvalue > 1e-4


def test_shared_window_containment():
    views = [ViewDesc(spatial_group=q, scale=(s, 1.0)) for q, s in enumerate((0.08, 0.2, 0.35, 0.5))]
    spec = _spec(views, shared_window=True)
    W, H = 1920, 1080
    for clip in range(500):
        m = oracle.ClipMeta()
        oracle.lib().oracle_spatial(ctypes.byref(spec), 0, clip, W, H, ctypes.byref(m))
        boxes = [list(m.box[q]) for q in range(4)]
        Wwin = max(b[2] for b in boxes)
        Hwin = max(b[3] for b in boxes)
        x_lo = min(b[0] for b in boxes)
        y_lo = min(b[1] for b in boxes)
        # all boxes fit one Wwin x Hwin window that lies inside the frame
        assert max(b[0] + b[2] for b in boxes) - x_lo <= Wwin
        assert max(b[1] + b[3] for b in boxes) - y_lo <= Hwin
        assert all(b[0] >= 0 and b[1] >= 0 and b[0] + b[2] <= W and b[1] + b[3] <= H for b in boxes)
        # the largest crop IS the window in its own dimension
        big = max(range(4), key=lambda q: boxes[q][2])
        assert boxes[big][2] == Wwin


def test_aug_gates_rates_and_ranges():
    v = ViewDesc(flip_p=0.5, rot_p=0.3, rot_max_deg=10.0, blur_p=0.7, sigma=(0.1, 2.0))
    spec = _spec([v])
    flips, rots, blurs, th, sg = [], [], [], [], []
    for clip in range(6000):
        m = oracle.ClipMeta()
        oracle.lib().oracle_spatial(ctypes.byref(spec), 0, clip, 340, 256, ctypes.byref(m))
        flips.append(m.flip[0]); rots.append(m.rot_on[0]); blurs.append(m.blur_on[0])
        th.append(m.theta[0]); sg.append(m.sigma[0])
    for obs, p in ((flips, 0.5), (rots, 0.3), (blurs, 0.7)):
        assert scipy.stats.binomtest(int(sum(obs)), len(obs), p).pvalue > 1e-4
    assert scipy.stats.kstest((np.array(th) + 10) / 20, "uniform").pvalue > 1e-4
    assert scipy.stats.kstest((np.array(sg) - 0.1) / 1.9, "uniform").pvalue > 1e-4


@pytest.mark.parametrize("sigma", [0.1, 0.3, 0.374, 0.376, 0.9, 1.37, 2.0, 2.6, 3.1])
def test_blur_radius_is_scipy_truncate_rule(sigma):
    # scipy.ndimage.gaussian_filter1d(truncate=4) support radius, measured on an impulse
    imp = np.zeros(101)
    imp[50] = 1.0
    resp = scipy.ndimage.gaussian_filter1d(imp, sigma, truncate=4.0, mode="mirror")
    r_scipy = int(np.max(np.nonzero(resp)[0]) - 50)
    spec = _spec([ViewDesc(blur_p=1.0, sigma=(sigma, sigma), blur_ksize=23, blur_truncate=4.0)])
    m = oracle.ClipMeta()
    oracle.lib().oracle_spatial(ctypes.byref(spec), 0, 0, 340, 256, ctypes.byref(m))
    assert m.blur_r[0] == min(11, r_scipy)


def test_same_seed_same_plan_other_epoch_differs():
    spec = _spec([ViewDesc(clip_len=16, stride=4)], batch_size=4)
    ds = oracle.make_dataset([(v, 300, 340, 256) for v in range(32)])
    a = oracle.plan_batch(spec, ds, 32, 5, 0, 2)
    b = oracle.plan_batch(spec, ds, 32, 5, 0, 2)
    c = oracle.plan_batch(spec, ds, 32, 6, 0, 2)
    da = [oracle.meta_to_dict(spec, m) for m in a]
    assert da == [oracle.meta_to_dict(spec, m) for m in b]
    assert da != [oracle.meta_to_dict(spec, m) for m in c]


def test_world_size_invariance_of_clip_plans():
    # R#1: counters use global clip ids, never the rank: a clip's plan is identical at W=1 and W=8
    spec1 = _spec([ViewDesc(clip_len=16, stride=4)], batch_size=4, world_size=1)
    spec8 = _spec([ViewDesc(clip_len=16, stride=4)], batch_size=4, world_size=8)
    ds = oracle.make_dataset([(100 + v, 300, 340, 256) for v in range(64)])
    by_clip = {}
    for it in range(oracle.iterations(spec1, 64)):
        for m in oracle.plan_batch(spec1, ds, 64, 0, 0, it):
            by_clip[m.clip] = oracle.meta_to_dict(spec1, m)
    seen = 0
    for r in range(8):
        for it in range(oracle.iterations(spec8, 64)):
            for m in oracle.plan_batch(spec8, ds, 64, 0, r, it):
                assert oracle.meta_to_dict(spec8, m) == by_clip[m.clip]
                seen += 1
    assert seen == 64


# ------------------------------------------------------------------ §8(f) f1: k-epoch shared frame pool

def _pool_meta(spec_desc, vids, epoch, clip):
    ospec = oracle.make_spec(spec_desc)
    ods = oracle.make_dataset(vids)
    ref = oracle.ClipMeta()
    oracle.lib().oracle_plan_clip(oracle.ctypes.byref(ospec), ods, epoch, clip, oracle.ctypes.byref(ref))
    return ref


def _k400_desc(k, views=None):
    views = views or [oracle.ViewDesc(clip_len=16, stride=4, out_h=224, out_w=224)]
    return oracle.SpecDesc(seed=11, batch_size=4, pool_epochs=k, views=views)


def test_k_epoch_pool_is_the_chunk_pool():
    """P:L270 (pool cached for exactly k epochs), R#25: with pool_epochs = k the pool start of
    epoch e is the start the per-epoch planner (k = 1) draws at epoch floor(e / k); k = 0 and
    k = 1 are the per-epoch planner itself."""
    vids = [(1000 + i, 300, 340, 256) for i in range(12)]
    for clip in range(12):
        for e in range(13):
            one = _pool_meta(_k400_desc(1), vids, e, clip)
            assert _pool_meta(_k400_desc(0), vids, e, clip).pool_start == one.pool_start
            for k in (2, 5):
                got = _pool_meta(_k400_desc(k), vids, e, clip)
                chunk = _pool_meta(_k400_desc(1), vids, e // k, clip)
                assert got.pool_start == chunk.pool_start
                assert list(got.frames[0][:16]) == list(chunk.frames[0][:16])   # single view: span == pool


def test_k_epoch_pool_keeps_per_epoch_offsets_and_spatial_draws():
    """Inside a chunk the pool is fixed, but a view shorter than the pool still draws its offset
    per epoch, and the spatial draws stay per epoch (randomness preserved)."""
    vids = [(1000 + i, 150, 1920, 1080) for i in range(16)]
    views = [oracle.ViewDesc(clip_len=16, stride=4, out_h=224, out_w=224),
             oracle.ViewDesc(clip_len=8, stride=4, out_h=224, out_w=224, spatial_group=1)]
    desc = _k400_desc(10, views)
    offsets_vary = boxes_vary = 0
    for clip in range(16):
        m = [_pool_meta(desc, vids, e, clip) for e in range(10)]
        assert len({x.pool_start for x in m}) == 1
        offsets_vary += len({x.frames[1][0] for x in m}) > 1
        boxes_vary += len({tuple(x.box[0]) for x in m}) > 1
    assert offsets_vary >= 12 and boxes_vary == 16


def test_k_epoch_pool_frame_reuse_over_ten_epochs():
    """Fig. 19 analogue on synthetic 300-frame videos, K400 clips (16 x stride 4):
    over ten epochs every selected frame is selected ten times with k = 10, while with fresh
    pools (k = 1) few frames are selected four or more times."""
    vids = [(1000 + i, 300, 340, 256) for i in range(64)]

    def counts(k):
        c = {}
        for e in range(10):
            for clip in range(64):
                m = _pool_meta(_k400_desc(k), vids, e, clip)
                for f in m.frames[0][:16]:
                    c[(m.video, f)] = c.get((m.video, f), 0) + 1
        return np.array(list(c.values()))

    c1, c10 = counts(1), counts(10)
    assert np.all(c10 == 10)
    assert np.mean(c1 >= 4) < 0.15


# ------------------------------------------------------------------ §8(f) f4: PySlowFast linspace slow pathway

def test_linspace_index_is_linspace_truncated():
    """R#26 pin: the oracle's index law is torch.linspace(0, n - 1, T) truncated, for every
    T, n <= 64: against float64 linspace wherever it is not within 1e-9 of an integer (there it
    must be that integer), and equal to PySlowFast's float32 torch.linspace(...).long() for the
    SlowFast 32 -> 8 selection."""
    L = oracle.lib()
    for n in range(1, 65):
        for T in range(1, 65):
            ref = torch.linspace(0, n - 1, T, dtype=torch.float64).tolist()
            for i in range(T):
                got = L.oracle_linspace_index(i, T, n)
                r = ref[i]
                assert got == (round(r) if abs(r - round(r)) < 1e-9 else math.floor(r)), (n, T, i)
    assert [L.oracle_linspace_index(i, 8, 32) for i in range(8)] == torch.linspace(0, 31, 8).long().tolist()


def test_slowfast_linspace_slow_is_fast_at_linspace_positions():
    from paper_conf_sosp_yelllhkh25_b200 import configs
    w = configs.slowfast_linspace()
    import sys
    import os
    sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
    from helpers import to_oracle
    ospec = to_oracle(w.spec)
    vids = [(1000 + i, 300, 340, 256) for i in range(8)]
    ods = oracle.make_dataset(vids)
    pos = torch.linspace(0, 31, 8).long().tolist()
    assert pos == [0, 4, 8, 13, 17, 22, 26, 31]
    for e in (0, 3):
        for clip in range(8):
            m = oracle.ClipMeta()
            oracle.lib().oracle_plan_clip(ctypes.byref(ospec), ods, e, clip, ctypes.byref(m))
            fast = list(m.frames[0][:32])
            assert list(m.frames[1][:8]) == [fast[p] for p in pos]
