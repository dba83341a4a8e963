"""Pin of oracle O13 (algorithmic source bytes) on
non-identity geometry.

O13 counts the distinct 32-byte sectors of (video, frame, plane, row) that the
bilinear taps of a batch touch. This test re-derives that number by brute force,
independently of the C oracle's separable row/column marking:

  * the taps of EVERY output pixel (the four (x, y) corners of R#12's bilinear
    interpolation) are enumerated one pixel at a time in numpy float32;
  * the tap rule itself is pinned to torch: for every output column / row, the
    source indices with a nonzero weight in ``torch.nn.functional.interpolate``
    (bilinear, align_corners=False, no antialias — R#12) are exactly {i0}, plus
    {i1} whenever lambda > 0 (i1 is read with weight 0 when lambda == 0, which the
    kernels and O13 both count as touched);
  * each touched pixel is mapped to byte ADDRESSES of a pitched NV12 frame (Y byte
    at y * pitch + x; U and V bytes at (y // 2) * pitch + 2 * (x // 2) + {0, 1}) and
    sectors are address // 32 — no per-plane sector formula is shared with O13.

A dropped i1 tap, a mis-mapped UV sector, a flipped/transposed axis or a missing
dedup across views fails one of the cases below (RRC up- and down-scaling,
short-side resize with real scaling, several groups sharing a frame, SlowFast
subsets).
"""
from __future__ import annotations

import numpy as np
import pytest
import torch
import torch.nn.functional as F

import oracle
from oracle import GEOM_RRC, GEOM_SHORTSIDE_CROP, SpecDesc, ViewDesc


def _taps_1d(sc: np.float32, off: int, n_out: int, lim: int):
    """R#12 tap (i0, i1, lambda) of each output index, float32 arithmetic written out."""
    out = []
    for o in range(n_out):
        s = np.float32(np.float32(sc) * np.float32(np.float32(off + o) + np.float32(0.5))) - np.float32(0.5)
        s = max(np.float32(s), np.float32(0.0))
        i0 = int(s)
        lam = np.float32(s) - np.float32(i0)
        out.append((i0, min(i0 + 1, lim - 1), float(lam)))
    return out


def _torch_support(n_in: int, n_out: int):
    """Nonzero-weight source indices of each output index of torch's bilinear resize."""
    eye = torch.eye(n_in, dtype=torch.float32).reshape(n_in, 1, 1, n_in)
    w = F.interpolate(eye, size=(1, n_out), mode="bilinear", align_corners=False, antialias=False)
    w = w.reshape(n_in, n_out).T           # [o, i]
    return [set(np.nonzero(w[o].numpy())[0].tolist()) for o in range(n_out)]


def _axis_taps(geom, box_lo, box_len, out_n, full_n, resized_n):
    """Absolute source taps along one axis, checked against torch's weights."""
    if geom == GEOM_RRC:
        sc = np.float32(np.float32(box_len) / np.float32(out_n))
        taps = _taps_1d(sc, 0, out_n, box_len)
        sup = _torch_support(box_len, out_n)
        for o, (i0, i1, lam) in enumerate(taps):
            assert sup[o] == ({i0} | ({i1} if lam > 0 else set())), (o, i0, i1, lam, sup[o])
        return [(box_lo + i0, box_lo + i1) for i0, i1, _ in taps]
    sc = np.float32(np.float32(full_n) / np.float32(resized_n))
    taps = _taps_1d(sc, box_lo, out_n, full_n)
    sup = _torch_support(full_n, resized_n)
    for o, (i0, i1, lam) in enumerate(taps):
        assert sup[box_lo + o] == ({i0} | ({i1} if lam > 0 else set()))
    return [(i0, i1) for i0, i1, _ in taps]


def _brute_sectors(spec_desc: SpecDesc, videos, epoch=0, rank=0, it=0):
    spec = oracle.make_spec(spec_desc)
    ds = oracle.make_dataset(videos)
    metas = oracle.plan_batch(spec, ds, len(videos), epoch, rank, it)
    dims = {v[0]: (v[2], v[3]) for v in videos}
    touched = {}            # (video, frame) -> set of (x, y)
    out_bytes, uses = 0, 0
    esize = {oracle.U8: 1, oracle.BF16: 2, oracle.F32: 4}
    for m in metas:
        W, H = dims[m.video]
        for k, v in enumerate(spec_desc.views):
            uses += v.clip_len
            out_bytes += v.clip_len * 3 * v.out_h * v.out_w * esize[v.out_dtype]
            box = list(m.box[v.spatial_group])
            if v.geom == GEOM_RRC:
                xs = _axis_taps(GEOM_RRC, box[0], box[2], v.out_w, W, 0)
                ys = _axis_taps(GEOM_RRC, box[1], box[3], v.out_h, H, 0)
            else:   # box = (x_off, y_off, W', H') in the resized frame
                xs = _axis_taps(GEOM_SHORTSIDE_CROP, box[0], 0, v.out_w, W, box[2])
                ys = _axis_taps(GEOM_SHORTSIDE_CROP, box[1], 0, v.out_h, H, box[3])
            pix = set()
            for oy in range(v.out_h):               # every output pixel, its four corners
                y0, y1 = ys[oy]
                for ox in range(v.out_w):
                    x0, x1 = xs[ox]
                    pix.update(((x0, y0), (x1, y0), (x0, y1), (x1, y1)))
            for t in range(v.clip_len):
                touched.setdefault((m.video, m.frames[k][t]), set()).update(pix)
    sectors = 0
    for (vid, _f), pix in touched.items():
        W, H = dims[vid]
        pitch = (W + 63) // 64 * 64
        ysec, uvsec = set(), set()
        for x, y in pix:
            ysec.add((y * pitch + x) // 32)
            base = (y // 2) * pitch + 2 * (x // 2)
            uvsec.add(base // 32)
            uvsec.add((base + 1) // 32)
        sectors += len(ysec) + len(uvsec)
    return sectors, out_bytes, len(touched), uses, spec, ds


CASES = {
    # RRC mixing up- and down-scaling on a small frame, flips on
    "rrc_small": (SpecDesc(seed=3, batch_size=2, views=[ViewDesc(clip_len=4, stride=2, out_h=40, out_w=48,
                                                                 scale=(0.1, 0.9))]),
                  [(1, 40, 96, 80), (2, 40, 96, 80)]),
    # two groups on the same frames (union across groups), one view downscaling 3x
    "rrc_two_groups": (SpecDesc(seed=11, batch_size=2, views=[
        ViewDesc(clip_len=3, stride=3, out_h=24, out_w=20, scale=(0.5, 1.0)),
        ViewDesc(clip_len=3, stride=3, spatial_group=1, out_h=56, out_w=64, scale=(0.05, 0.3))]),
        [(5, 30, 128, 72), (6, 30, 128, 72)]),
    # short-side resize with real scaling on both axes (W' = 85 from 160x120, S = 64)
    "shortside_scaled": (SpecDesc(seed=7, batch_size=2, views=[ViewDesc(
        clip_len=4, stride=2, geom=GEOM_SHORTSIDE_CROP, short_side=64, out_h=56, out_w=56)]),
        [(9, 50, 160, 120), (10, 50, 160, 120)]),
    # SlowFast pathways: slow frames are a subset of the fast frames (dedup across views)
    "slowfast_subset": (SpecDesc(seed=1, batch_size=1, views=[
        ViewDesc(clip_len=8, stride=2, pool_offset=0, geom=GEOM_SHORTSIDE_CROP, short_side=48, out_h=40, out_w=40),
        ViewDesc(clip_len=2, stride=8, pool_offset=0, geom=GEOM_SHORTSIDE_CROP, short_side=48, out_h=40, out_w=40)]),
        [(4, 60, 100, 70)]),
}


@pytest.mark.parametrize("name", sorted(CASES))
def test_batch_bytes_brute_force(name):
    sd, videos = CASES[name]
    sectors, out_bytes, fetches, uses, spec, ds = _brute_sectors(sd, videos)
    r = oracle.batch_bytes(spec, ds, len(videos), 0, 0, 0)
    assert r.out_bytes == out_bytes
    assert r.fetches == fetches and r.uses == uses
    assert r.src_sectors == sectors, (r.src_sectors, sectors)


def test_brute_force_detects_a_dropped_tap():
    """The brute force is sensitive to the i1 tap: dropping it changes the sector count
    on a non-identity case (so the equality above is not vacuous)."""
    sd, videos = CASES["rrc_small"]
    full, *_ = _brute_sectors(sd, videos)
    global _taps_1d
    keep = _taps_1d
    try:
        _taps_1d = lambda sc, off, n, lim: [(i0, i0, lam) for i0, _i1, lam in keep(sc, off, n, lim)]  # noqa: E731
        try:
            dropped, *_ = _brute_sectors(sd, videos)
        except AssertionError:      # the torch support check already rejects the mutant
            return
    finally:
        _taps_1d = keep
    assert dropped < full
