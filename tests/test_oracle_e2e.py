"""End-to-end pins of the oracle on the tiny config (BASELINE.json configs[0]) and
closed forms for its byte / reuse accounting (O13, O14).

The whole oracle batch is compared with a pipeline composed from the paper's
op library (OpenCV colour conversion, torch bilinear interpolation in float64,
torch.flip, torchvision rotate / gaussian_blur, torchvision normalize) driven by
the oracle's (separately pinned) plan.
"""
import ctypes

import cv2
import numpy as np
import pytest
import torch
import torch.nn.functional as Fnn
import torchvision.transforms.functional as TF

import oracle
import synth
from oracle import SpecDesc, ViewDesc

TINY = SpecDesc(seed=0, batch_size=1, views=[ViewDesc(clip_len=8, stride=2, out_h=32, out_w=32, flip_p=0.5,
                                                      out_dtype=oracle.U8)])


def _frame_refs(metas, spec, videos, family, seed):
    refs, keep = [], []
    need = sorted({(m.video, m.frames[k][t]) for m in metas for k in range(spec.n_views)
                   for t in range(spec.views[k].clip_len)})
    dims = {v: (W, H) for v, F, W, H in videos}
    arr = (oracle.FrameRef * len(need))()
    for i, (v, f) in enumerate(need):
        W, H = dims[v]
        y, uv = synth.frames(family, seed, v, f, 1, W, H)
        keep += [y, uv]
        arr[i].video, arr[i].frame, arr[i].width, arr[i].height = v, f, W, H
        arr[i].y, arr[i].uv, arr[i].y_pitch, arr[i].uv_pitch = y.ctypes.data, uv.ctypes.data, W, W
    return arr, keep


def _library_pipeline(y, uv, box, flip, Ho, Wo):
    rgb = cv2.cvtColor(np.concatenate([y, uv], 0), cv2.COLOR_YUV2RGB_NV12)
    x0, y0, w, h = box
    crop = torch.from_numpy(np.ascontiguousarray(rgb[y0:y0 + h, x0:x0 + w])).permute(2, 0, 1)[None].double()
    r = Fnn.interpolate(crop, size=(Ho, Wo), mode="bilinear", align_corners=False, antialias=False)[0]
    if flip:
        r = torch.flip(r, dims=[2])
    return r.numpy()        # exact (float64) values before the uint8 quantisation


@pytest.mark.parametrize("family", [synth.UNIFORM, synth.SMOOTH])
@pytest.mark.parametrize("epoch", [0, 1, 2, 3])
def test_tiny_batch_vs_library_pipeline(family, epoch):
    spec = oracle.make_spec(TINY)
    videos = [(0, 16, 64, 64)]
    ds = oracle.make_dataset(videos)
    metas = oracle.plan_batch(spec, ds, 1, epoch, 0, 0)
    refs, keep = _frame_refs(metas, spec, videos, family, 1)
    out = np.zeros((1, 3, 8, 32, 32), np.uint8)
    oracle.materialize(spec, ds, 1, epoch, 0, 0, refs, [out])
    m = metas[0]
    for t in range(8):
        y, uv = synth.frames(family, 1, 0, m.frames[0][t], 1, 64, 64)
        exact = _library_pipeline(y[0], uv[0], list(m.box[0]), m.flip[0], 32, 32)
        assert np.abs(out[0, :, t].astype(np.float64) - exact).max() <= 0.5 + 1e-3


def test_tiny_dtypes_agree_with_normalize():
    base = oracle.make_spec(TINY)
    videos = [(0, 16, 64, 64)]
    ds = oracle.make_dataset(videos)
    metas = oracle.plan_batch(base, ds, 1, 0, 0, 0)
    refs, keep = _frame_refs(metas, base, videos, synth.UNIFORM, 1)
    outs = {}
    for dt, npdt in ((oracle.U8, np.uint8), (oracle.BF16, np.uint16), (oracle.F32, np.float32)):
        sd = SpecDesc(seed=0, batch_size=1, views=[ViewDesc(clip_len=8, stride=2, out_h=32, out_w=32,
                                                            out_dtype=dt)])
        spec = oracle.make_spec(sd)
        o = np.zeros((1, 3, 8, 32, 32), npdt)
        oracle.materialize(spec, ds, 1, 0, 0, 0, refs, [o])
        outs[dt] = o
    mean, std = np.array(TINY.views[0].mean), np.array(TINY.views[0].std)
    ref = (outs[oracle.U8] / 255.0 - mean[None, :, None, None, None]) / std[None, :, None, None, None]
    assert np.abs(outs[oracle.F32] - ref).max() <= 1e-6
    bf = torch.from_numpy(outs[oracle.F32]).to(torch.bfloat16).view(torch.int16).numpy().astype(np.uint16)
    assert np.array_equal(outs[oracle.BF16], bf)


def test_two_view_rotate_blur_vs_library():
    sd = SpecDesc(seed=4, batch_size=2, views=[
        ViewDesc(clip_len=4, stride=4, spatial_group=0, out_h=64, out_w=64, rot_p=1.0, rot_max_deg=10.0,
                 blur_p=1.0, out_dtype=oracle.U8),
        ViewDesc(clip_len=4, stride=4, spatial_group=1, out_h=64, out_w=64, rot_p=0.0, blur_p=1.0,
                 out_dtype=oracle.U8)])
    spec = oracle.make_spec(sd)
    videos = [(5, 40, 96, 80), (6, 40, 96, 80)]
    ds = oracle.make_dataset(videos)
    metas = oracle.plan_batch(spec, ds, 2, 0, 0, 0)
    refs, keep = _frame_refs(metas, spec, videos, synth.SMOOTH, 2)
    outs = [np.zeros((2, 3, 4, 64, 64), np.uint8) for _ in range(2)]
    oracle.materialize(spec, ds, 2, 0, 0, 0, refs, outs)
    for b, m in enumerate(metas):
        assert m.frames[0][:4] == m.frames[1][:4]          # views share the clip (R#6)
        for k in range(2):
            q = k
            for t in range(4):
                y, uv = synth.frames(synth.SMOOTH, 2, m.video, m.frames[k][t], 1, 96, 80)
                stage = np.round(_library_pipeline(y[0], uv[0], list(m.box[q]), m.flip[q], 64, 64))
                img = torch.from_numpy(stage).float()
                if m.rot_on[q]:
                    img = torch.round(TF.rotate(img, m.theta[q], interpolation=TF.InterpolationMode.BILINEAR))
                r = m.blur_r[q]
                if m.blur_on[q] and r > 0:
                    img = torch.round(TF.gaussian_blur(img, [2 * r + 1] * 2, [m.sigma[q]] * 2))
                d = np.abs(outs[k][b, :, t].astype(np.int32) - img.numpy().astype(np.int32))
                # each quantised stage may flip a rounding tie: allow 1 LSB per stage (<= 3)
                assert d.max() <= 3
                assert (d > 1).mean() < 0.01


def test_batch_bytes_closed_forms():
    # identity geometry (crop = whole frame, out = frame size): every pixel is a tap
    W, H, T = 96, 64, 4
    sd = SpecDesc(seed=0, batch_size=2, views=[ViewDesc(clip_len=T, stride=1, out_h=H, out_w=W,
                                                        scale=(1.0, 1.0), ratio=(1.5, 1.5), flip_p=0.0)])
    spec = oracle.make_spec(sd)
    ds = oracle.make_dataset([(0, 50, W, H), (1, 50, W, H)])
    r = oracle.batch_bytes(spec, ds, 2, 0, 0, 0)
    sectors_per_frame = H * ((W + 31) // 32) + (H // 2) * ((W + 31) // 32)
    assert r.fetches == 2 * T and r.uses == 2 * T
    assert r.src_sectors == 2 * T * sectors_per_frame
    assert r.out_bytes == 2 * T * 3 * H * W * 2
    # SlowFast-style pathways: slow frames are a subset of fast frames -> fetches count fast only
    sd = SpecDesc(seed=0, batch_size=1, views=[
        ViewDesc(clip_len=32, stride=2, pool_offset=0, out_h=32, out_w=32),
        ViewDesc(clip_len=8, stride=8, pool_offset=0, out_h=32, out_w=32)])
    spec = oracle.make_spec(sd)
    r = oracle.batch_bytes(spec, oracle.make_dataset([(3, 300, 64, 64)]), 1, 0, 0, 0)
    assert r.fetches == 32 and r.uses == 40
