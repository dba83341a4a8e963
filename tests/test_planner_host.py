"""CPU parity of the product's host planner (libsand.so, no device) against the oracle.

The plan (clip order per rank, frame indices, crop boxes, flip/rotation/blur draws) is the
integer/double part of the path (§8(a) rows a1-a3); it must be BIT-EXACT (north_star). These
tests call the host-only C-ABI entry points sand_plan_rank_clips / sand_plan_clip, which share
the planner read_batch uses; the GPU tests check the same through sand_view_get_meta.
"""
import numpy as np
import pytest

import oracle
import paper_conf_sosp_yelllhkh25_b200 as sand
from paper_conf_sosp_yelllhkh25_b200 import configs

from helpers import meta_fields, to_oracle, videos_of


@pytest.mark.parametrize("name", ["tiny", "k400", "slowfast", "twoview", "ray"])
def test_host_plan_matches_oracle_bit_exact(name):
    w = configs.get(name)
    vids = videos_of(w, min(w.n_videos, 64))
    ospec = to_oracle(w.spec)
    ods = oracle.make_dataset(vids)
    rng = np.random.default_rng(3)
    n = len(vids) * w.spec.samples_per_video
    for epoch in (0, 1, 7, 2**33 + 5):
        for clip in rng.choice(n, size=min(n, 24), replace=False):
            got = sand.plan_clip(w.spec, vids, epoch, int(clip))
            ref = oracle.ClipMeta()
            oracle.lib().oracle_plan_clip(oracle.ctypes.byref(ospec), ods, epoch, int(clip), oracle.ctypes.byref(ref))
            assert meta_fields(w.spec, got) == meta_fields(w.spec, ref), (name, epoch, clip)


@pytest.mark.parametrize("n_videos,world,drop_last,S", [(64, 1, False, 1), (64, 8, False, 1), (70, 8, False, 1),
                                                       (70, 8, True, 1), (5, 8, False, 1), (33, 4, False, 2)])
def test_rank_clips_match_oracle_partition(n_videos, world, drop_last, S):
    spec = configs.k400().spec
    spec.world_size, spec.drop_last, spec.samples_per_video = world, drop_last, S
    vids = [1000 + i for i in range(n_videos)]
    for epoch in (0, 3):
        perm = oracle.permutation(n_videos * S, spec.seed, epoch)
        for r in range(world):
            assert sand.plan_rank_clips(spec, vids, epoch, r) == oracle.partition(perm, world, r, drop_last).tolist()


def test_samples_per_video_and_shared_window_plans():
    w = configs.ray()
    w.spec.samples_per_video = 2
    vids = videos_of(w, 8)
    ospec = to_oracle(w.spec)
    ods = oracle.make_dataset(vids)
    for clip in range(16):
        got = sand.plan_clip(w.spec, vids, 4, clip)
        ref = oracle.ClipMeta()
        oracle.lib().oracle_plan_clip(oracle.ctypes.byref(ospec), ods, 4, clip, oracle.ctypes.byref(ref))
        assert meta_fields(w.spec, got) == meta_fields(w.spec, ref)
        assert got.sample == clip % 2


def test_invalid_specs_rejected_on_host():
    w = configs.tiny()
    vids = videos_of(w)
    bad = configs.tiny().spec
    bad.views[0].blur_ksize = 22
    with pytest.raises(sand.SandError):
        sand.plan_clip(bad, vids, 0, 0)
    bad = configs.tiny().spec
    bad.views[0].clip_len = 0
    with pytest.raises(sand.SandError):
        sand.plan_rank_clips(bad, [1000], 0, 0)
    two = configs.twoview().spec
    two.views[1].rot_max_deg = 3.0
    two.views[1].spatial_group = 0           # same group, different augmentation -> invalid
    with pytest.raises(sand.SandError):
        sand.plan_clip(two, videos_of(configs.twoview(), 4), 0, 0)


@pytest.mark.parametrize("name,k", [("k400", 4), ("slowfast", 10), ("ray", 3)])
def test_host_plan_k_epoch_pool_matches_oracle(name, k):
    """§8(f) f1: with pool_epochs = k the host planner still matches the oracle bit-exactly."""
    w = configs.get(name)
    w.spec.pool_epochs = k
    vids = videos_of(w, min(w.n_videos, 32))
    ospec = to_oracle(w.spec)
    ods = oracle.make_dataset(vids)
    for epoch in (0, k - 1, k, 3 * k + 1):
        for clip in range(0, len(vids), 3):
            got = sand.plan_clip(w.spec, vids, epoch, clip)
            ref = oracle.ClipMeta()
            oracle.lib().oracle_plan_clip(oracle.ctypes.byref(ospec), ods, epoch, clip, oracle.ctypes.byref(ref))
            assert meta_fields(w.spec, got) == meta_fields(w.spec, ref), (name, k, epoch, clip)


def test_host_plan_linspace_slow_pathway_matches_oracle():
    """§8(f) f4 (R#26): the linspace slow pathway plans bit-exactly like the oracle."""
    w = configs.slowfast_linspace()
    vids = videos_of(w, 16)
    ospec = to_oracle(w.spec)
    ods = oracle.make_dataset(vids)
    for epoch in (0, 2, 9):
        for clip in range(16):
            got = sand.plan_clip(w.spec, vids, epoch, clip)
            ref = oracle.ClipMeta()
            oracle.lib().oracle_plan_clip(oracle.ctypes.byref(ospec), ods, epoch, clip, oracle.ctypes.byref(ref))
            assert meta_fields(w.spec, got) == meta_fields(w.spec, ref), (epoch, clip)
    bad = configs.slowfast_linspace().spec
    bad.views[0].subsample_of = 1            # a sub-sample of a sub-sample
    with pytest.raises(sand.SandError):
        sand.plan_clip(bad, vids, 0, 0)


def _plan_equal(spec, vids, epochs, clips):
    ospec = to_oracle(spec)
    ods = oracle.make_dataset(vids)
    for epoch in epochs:
        for clip in clips:
            got = sand.plan_clip(spec, vids, epoch, clip)
            ref = oracle.ClipMeta()
            oracle.lib().oracle_plan_clip(oracle.ctypes.byref(ospec), ods, epoch, clip, oracle.ctypes.byref(ref))
            assert meta_fields(spec, got) == meta_fields(spec, ref), (epoch, clip)
            yield got


def test_host_plan_short_video_clamp_matches_oracle():
    """Videos shorter than the shared pool (F < P, R#4): start 0 and indices clamped to F - 1."""
    w = configs.slowfast()
    vids = [(1000 + i, 20 + 7 * i, 340, 256) for i in range(6)]     # F in 20..55 < P = 63
    for got in _plan_equal(w.spec, vids, (0, 3), range(6)):
        F = vids[got.clip][1]
        assert got.pool_start == 0 and max(got.frames[0][:32]) == F - 1


def test_host_plan_rrc_central_fallback_matches_oracle():
    """An RRC range no attempt satisfies takes torchvision's central fallback (R#8), in both
    directions of the ratio clamp."""
    for ratio, box in (((2.5, 3.0), [0, 60, 340, 136]), ((0.2, 0.25), [138, 0, 64, 256])):
        spec = configs.Spec(batch_size=1, views=[configs.ViewSpec(clip_len=4, stride=2, scale=(0.95, 1.0),
                                                                  ratio=ratio)])
        vids = [(1000 + i, 30, 340, 256) for i in range(4)]
        for got in _plan_equal(spec, vids, (0, 1, 5), range(4)):
            assert list(got.box[0]) == box


def test_host_plan_color_jitter_draws_match_oracle():
    """f4 (R#30): colour-jitter gates, factors and op orders plan bit-exactly like the oracle."""
    w = configs.twoview()
    for v in w.spec.views:
        v.jitter_p, v.brightness, v.contrast, v.saturation = 0.8, 0.4, 0.4, 0.4
    vids = videos_of(w, 16)
    got = list(_plan_equal(w.spec, vids, (0, 3), range(16)))
    on = [m.jitter_on[q] for m in got for q in (0, 1)]
    assert 0 < sum(on) < len(on)
    assert all(0.6 <= m.jitter_f[q][i] <= 1.4 for m in got for q in (0, 1) for i in range(3))
    assert {m.jitter_order[q] for m in got for q in (0, 1)} == set(range(6))
