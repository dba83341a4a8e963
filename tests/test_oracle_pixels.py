"""Pins for the oracle's pixel stages (O6-O11) against the paper's op library.

The paper's engine runs its augmentation with OpenCV and libtorch, so
each stage is pinned to those libraries: NV12->RGB exhaustively against
cv2.cvtColor(COLOR_YUV2RGB_NV12); bilinear resample against torch
F.interpolate and, on 4x4 frames, against the exact float64 result for every
crop box; flip against torch.flip; rotation against torchvision F.rotate;
blur against scipy.ndimage.gaussian_filter1d and torchvision gaussian_blur;
normalisation against torchvision normalize and torch's bfloat16 cast. The
bound "within 1 LSB" is the north_star's uint8 tolerance; the oracle's fp32
result must also lie within 0.5 + 1e-3 of the exact value where one exists.
"""
import math

import cv2
import numpy as np
import pytest
import scipy.ndimage
import torch
import torch.nn.functional as Fnn
import torchvision.transforms.functional as TF

import oracle
import synth

RNG = np.random.default_rng(20251013)


# ---------------------------------------------------------------- O6 NV12 -> RGB

def test_nv12_to_rgb_exhaustive_vs_opencv():
    # every (Y, U, V) triple: chroma grid 4096 x 1024 = 2^22 samples = 2^16 (U,V) pairs x 64 blocks,
    # each 2x2 luma block of a chroma sample carries 4 of the 256 Y values
    Wc, Hc = 4096, 1024
    idx = np.arange(Wc * Hc, dtype=np.int64).reshape(Hc, Wc)
    uvpair = idx % 65536
    block = idx // 65536                       # 0..63 -> Y values block*4 .. block*4+3
    U = (uvpair // 256).astype(np.uint8)
    V = (uvpair % 256).astype(np.uint8)
    Y = np.empty((2 * Hc, 2 * Wc), np.uint8)
    base = (block * 4).astype(np.uint8)
    Y[0::2, 0::2] = base
    Y[0::2, 1::2] = base + 1
    Y[1::2, 0::2] = base + 2
    Y[1::2, 1::2] = base + 3
    uv = np.empty((Hc, 2 * Wc), np.uint8)
    uv[:, 0::2] = U
    uv[:, 1::2] = V
    ours = oracle.nv12_to_rgb(Y, uv)
    ref = cv2.cvtColor(np.concatenate([Y, uv], axis=0), cv2.COLOR_YUV2RGB_NV12)
    assert ours.shape == ref.shape
    assert np.array_equal(ours, ref)


def test_nv12_synthetic_frames_vs_opencv():
    for fam in (synth.UNIFORM, synth.SMOOTH):
        y, uv = synth.frames(fam, 3, 9, 17, 1, 340, 256)
        ref = cv2.cvtColor(np.concatenate([y[0], uv[0]], axis=0), cv2.COLOR_YUV2RGB_NV12)
        assert np.array_equal(oracle.nv12_to_rgb(y[0], uv[0]), ref)


# ---------------------------------------------------------------- O7 bilinear resample

def _torch_resize(img, Ho, Wo, dtype=torch.float32):
    t = torch.from_numpy(img).to(dtype).permute(2, 0, 1)[None]
    r = Fnn.interpolate(t, size=(Ho, Wo), mode="bilinear", align_corners=False, antialias=False)
    return r[0].permute(1, 2, 0)


@pytest.mark.parametrize("h,w,Ho,Wo", [(256, 340, 224, 224), (70, 90, 224, 224), (256, 200, 112, 160),
                                       (13, 7, 32, 32), (1080, 1920, 224, 224), (33, 65, 33, 65)])
def test_resize_vs_torch_interpolate(h, w, Ho, Wo):
    img = RNG.integers(0, 256, (h, w, 3), dtype=np.uint8)
    ours = oracle.resize(img, Ho, Wo).astype(np.int32)
    ref32 = torch.round(_torch_resize(img, Ho, Wo)).numpy().astype(np.int32)
    d = np.abs(ours - ref32)
    assert d.max() <= 1
    assert (d > 0).mean() < 2e-3
    exact = _torch_resize(img, Ho, Wo, torch.float64).numpy()
    assert np.abs(ours - exact).max() <= 0.5 + _coord_slack(max(h, w))


def _coord_slack(n):
    # fp32 source coordinates carry <= 3 roundings of a value <= n per axis (R#12): the
    # lerp weight error is <= 3 * n * 2^-24, times a pixel step of at most 255, two axes,
    # plus three rounded lerp ops on values <= 255
    return 2 * 255 * 3 * n * 2.0 ** -24 + 3 * 255 * 2.0 ** -24


def test_resize_identity_constant_gradient():
    img = RNG.integers(0, 256, (57, 91, 3), dtype=np.uint8)
    assert np.array_equal(oracle.resize(img, 57, 91), img)            # identity size -> input
    const = np.full((40, 50, 3), 137, np.uint8)
    assert (oracle.resize(const, 224, 224) == 137).all()              # constant stays constant
    # linear gradient, 2x upscale: taps weights 1/4, 3/4 on a step-4 ramp -> integers, exact inside
    ramp = (np.arange(32) * 4).astype(np.uint8)
    g = np.broadcast_to(ramp[None, :, None], (8, 32, 3)).copy()
    up = oracle.resize(g, 8, 64)[0, :, 0].astype(np.int32)
    interior = [(2 * ox + 1) - 1 + 0.5 for ox in range(1, 63)]    # 4 * (ox/2 - 1/4) = 2*ox - 1
    assert up[1:63].tolist() == [2 * ox - 1 for ox in range(1, 63)]
    assert up[0] == 0 and up[63] == 124                             # half-pixel clamp at the borders


def test_resized_crop_4x4_all_boxes_bruteforce():
    # every crop box of a 4x4 frame x both flips x output sizes 1..8: oracle vs the exact value
    img = RNG.integers(0, 256, (4, 4, 3), dtype=np.uint8)
    for y0 in range(4):
        for x0 in range(4):
            for h in range(1, 5 - y0):
                for w in range(1, 5 - x0):
                    crop = img[y0:y0 + h, x0:x0 + w]
                    for Ho in range(1, 9):
                        Wo = 9 - Ho
                        ours = oracle.resized_crop(img, (x0, y0, w, h), Ho, Wo).astype(np.int32)
                        exact = _torch_resize(np.ascontiguousarray(crop), Ho, Wo, torch.float64).numpy()
                        assert np.abs(ours - exact).max() <= 0.5 + _coord_slack(8)
                        fl = oracle.flip(oracle.resized_crop(img, (x0, y0, w, h), Ho, Wo))
                        assert np.array_equal(fl, ours[:, ::-1].astype(np.uint8))


def test_shortside_crop_is_resize_then_crop():
    img = RNG.integers(0, 256, (720, 1280, 3), dtype=np.uint8)
    box = (101, 17, 455, 256)              # x_off, y_off, W', H'
    full = _torch_resize(img, 256, 455, torch.float64).numpy()
    ours = oracle.shortside_crop(img, box, 224, 224).astype(np.int32)
    assert np.abs(ours - full[17:17 + 224, 101:101 + 224]).max() <= 0.5 + _coord_slack(1280)
    # identity short side: a pure copy of the crop
    img2 = RNG.integers(0, 256, (256, 340, 3), dtype=np.uint8)
    assert np.array_equal(oracle.shortside_crop(img2, (50, 20, 340, 256), 224, 224),
                          img2[20:244, 50:274])


# ---------------------------------------------------------------- O8 flip

def test_flip_vs_torch_flip_and_involution():
    img = RNG.integers(0, 256, (31, 45, 3), dtype=np.uint8)
    ref = torch.flip(torch.from_numpy(img), dims=[1]).numpy()
    assert np.array_equal(oracle.flip(img), ref)
    assert np.array_equal(oracle.flip(oracle.flip(img)), img)


# ---------------------------------------------------------------- O9 rotation

@pytest.mark.parametrize("theta", [-10.0, -3.7, 0.5, 4.2, 9.99, 30.0])
def test_rotate_vs_torchvision(theta):
    img = RNG.integers(0, 256, (224, 224, 3), dtype=np.uint8)
    t = torch.from_numpy(img).permute(2, 0, 1).float()
    ref = TF.rotate(t, theta, interpolation=TF.InterpolationMode.BILINEAR, fill=None)
    ref = torch.round(ref).permute(1, 2, 0).numpy().astype(np.int32)
    ours = oracle.rotate(img, theta).astype(np.int32)
    d = np.abs(ours - ref)
    assert d.max() <= 1
    assert (d > 0).mean() < 5e-3


def test_rotate_zero_is_identity_and_rect():
    img = RNG.integers(0, 256, (32, 48, 3), dtype=np.uint8)
    assert np.array_equal(oracle.rotate(img, 0.0), img)
    t = torch.from_numpy(img).permute(2, 0, 1).float()
    ref = torch.round(TF.rotate(t, 7.0, interpolation=TF.InterpolationMode.BILINEAR)).permute(1, 2, 0)
    assert np.abs(oracle.rotate(img, 7.0).astype(np.int32) - ref.numpy().astype(np.int32)).max() <= 1


def test_rotate_constant_interior_preserved():
    img = np.full((64, 64, 3), 200, np.uint8)
    r = oracle.rotate(img, 8.0)
    assert (r[16:48, 16:48] == 200).all()
    assert r[0, 0, 0] < 200                   # a corner samples the zero fill


# ---------------------------------------------------------------- O10 blur

def _scipy_blur(img, sigma):
    f = img.astype(np.float64)
    f = scipy.ndimage.gaussian_filter1d(f, sigma, axis=1, mode="mirror", truncate=4.0)
    f = scipy.ndimage.gaussian_filter1d(f, sigma, axis=0, mode="mirror", truncate=4.0)
    return f


@pytest.mark.parametrize("sigma", [0.1, 0.5, 1.0, 1.37, 2.0])
def test_blur_vs_scipy_and_torchvision(sigma):
    img = RNG.integers(0, 256, (224, 224, 3), dtype=np.uint8)
    r = min(11, int(math.floor(4.0 * sigma + 0.5)))
    ours = oracle.blur(img, sigma, r).astype(np.int32)
    ref = _scipy_blur(img, sigma)
    assert np.abs(ours - ref).max() <= 0.5 + 2e-3
    assert np.abs(ours - np.round(ref)).max() <= 1
    if r >= 1:
        t = torch.from_numpy(img).permute(2, 0, 1).float()
        tv = TF.gaussian_blur(t, [2 * r + 1, 2 * r + 1], [sigma, sigma])
        tv = torch.round(tv).permute(1, 2, 0).numpy().astype(np.int32)
        assert np.abs(ours - tv).max() <= 1


def test_blur_weights_sum_and_symmetry():
    w = oracle.blur_weights(1.3, 5)
    assert len(w) == 11
    assert abs(float(np.sum(w.astype(np.float64))) - 1.0) < 1e-6
    assert np.array_equal(w, w[::-1])
    assert np.argmax(w) == 5


def test_blur_constant_stays_constant():
    img = np.full((40, 40, 3), 77, np.uint8)
    assert (oracle.blur(img, 2.0, 8) == 77).all()


# ---------------------------------------------------------------- O11 normalise

def test_normalize_vs_torchvision_and_bf16():
    mean, std = (0.485, 0.456, 0.406), (0.229, 0.224, 0.225)
    q = RNG.integers(0, 256, (16, 16, 3), dtype=np.uint8)
    f32 = oracle.normalize(q, mean, std, oracle.F32)
    t = torch.from_numpy(q).permute(2, 0, 1).double() / 255.0
    ref = TF.normalize(t, mean, std).numpy()
    assert np.abs(f32 - ref).max() <= 1e-6
    bf = oracle.normalize(q, mean, std, oracle.BF16)
    ref_bf = torch.from_numpy(f32).to(torch.bfloat16).view(torch.int16).numpy().astype(np.uint16)
    assert np.array_equal(bf, ref_bf)
    # every u8 value for one channel
    a, b = oracle.norm_coeffs(mean, std)
    L = oracle.lib()
    vals = np.array([L.oracle_normalize(i, float(a[0]), float(b[0])) for i in range(256)], np.float32)
    assert np.abs(vals - (np.arange(256) / 255.0 - mean[0]) / std[0]).max() <= 1e-6


def _all_triples():
    Wc, Hc = 4096, 1024
    idx = np.arange(Wc * Hc, dtype=np.int64).reshape(Hc, Wc)
    uvpair = idx % 65536
    block = idx // 65536
    U = (uvpair // 256).astype(np.uint8)
    V = (uvpair % 256).astype(np.uint8)
    Y = np.empty((2 * Hc, 2 * Wc), np.uint8)
    base = (block * 4).astype(np.uint8)
    Y[0::2, 0::2] = base
    Y[0::2, 1::2] = base + 1
    Y[1::2, 0::2] = base + 2
    Y[1::2, 1::2] = base + 3
    uv = np.empty((Hc, 2 * Wc), np.uint8)
    uv[:, 0::2] = U
    uv[:, 1::2] = V
    Uf = np.repeat(np.repeat(U, 2, axis=0), 2, axis=1).astype(np.float64)
    Vf = np.repeat(np.repeat(V, 2, axis=0), 2, axis=1).astype(np.float64)
    return Y, uv, Y.astype(np.float64), Uf, Vf


def test_bt709_exhaustive_vs_itu_matrix():
    """f4 (R#29): the BT.709 integer form against the ITU-R BT.709 matrix computed in float64
    from Kr = 0.2126, Kb = 0.0722 with the limited-range scales 255/219 and 255/224 (the
    standard's definition, not the oracle's constants): within 1 LSB for every (Y, U, V) with
    Y >= 16, identical in > 99.8 % of them; below 16 luma clamps like OpenCV's BT.601 form."""
    Y, uv, Yf, Uf, Vf = _all_triples()
    ours = oracle.nv12_to_rgb(Y, uv, 1).astype(np.int32)
    Kr, Kb = 0.2126, 0.0722
    Kg = 1 - Kr - Kb
    sy, sc = 255.0 / 219.0, 255.0 / 224.0
    yl = sy * (np.maximum(Yf, 16) - 16)
    u, v = Uf - 128, Vf - 128
    ref = np.stack([yl + 2 * (1 - Kr) * sc * v,
                    yl - 2 * Kb * (1 - Kb) / Kg * sc * u - 2 * Kr * (1 - Kr) / Kg * sc * v,
                    yl + 2 * (1 - Kb) * sc * u], axis=-1)
    ref = np.clip(np.floor(ref + 0.5), 0, 255).astype(np.int32)
    d = np.abs(ours - ref)
    assert d.max() <= 1
    assert (d == 0).mean() > 0.998
    # BT.709 differs from BT.601 (not a relabelled 601): most saturated colours change
    assert (ours != oracle.nv12_to_rgb(Y, uv, 0)).any(axis=-1).mean() > 0.5
    # Y < 16 behaves as Y = 16 (the clamp of the integer form)
    lo = Y < 16
    Y16 = np.where(lo, 16, Y).astype(np.uint8)
    assert np.array_equal(ours[lo], oracle.nv12_to_rgb(Y16, uv, 1).astype(np.int32)[lo])


def test_color_jitter_vs_torchvision():
    """f4 (R#30): the oracle's colour jitter against torchvision's adjust_brightness /
    adjust_contrast / adjust_saturation on uint8 tensors (the ops ColorJitter applies), one op at
    a time (within 1 LSB, identical for > 99 % of values) and composed in each of the 6 orders
    (within 1 LSB per stage); factor 1 is the identity."""
    import torch
    from torchvision.transforms.v2 import functional as TF
    rng = np.random.default_rng(11)
    ops = [TF.adjust_brightness, TF.adjust_contrast, TF.adjust_saturation]
    perms = [(0, 1, 2), (0, 2, 1), (1, 0, 2), (1, 2, 0), (2, 0, 1), (2, 1, 0)]
    diffs, composed = [], []
    for trial in range(24):
        img = rng.integers(0, 256, size=(40, 56, 3), dtype=np.uint8)
        if trial % 3 == 0:                               # natural-image-like smooth content
            img = np.clip(np.cumsum(rng.integers(-3, 4, size=(40, 56, 3)), axis=1) + 128, 0, 255).astype(np.uint8)
        f = rng.uniform(0.6, 1.4, size=3)
        order = trial % 6
        ours = oracle.color_jitter(img, f, order)
        t = torch.from_numpy(img).permute(2, 0, 1).contiguous()
        for op in perms[order]:
            t = ops[op](t, float(f[op]))
        ref = t.permute(1, 2, 0).numpy()
        composed.append(np.abs(ours.astype(int) - ref.astype(int)))
        for op in range(3):                              # each op alone (the others at factor 1)
            g = np.ones(3)
            g[op] = f[op]
            one = oracle.color_jitter(img, g, 0)
            r1 = ops[op](torch.from_numpy(img).permute(2, 0, 1).contiguous(), float(f[op])).permute(1, 2, 0).numpy()
            diffs.append(np.abs(one.astype(int) - r1.astype(int)))
        assert np.array_equal(oracle.color_jitter(img, [1.0, 1.0, 1.0], order), img)
    d = np.concatenate([x.ravel() for x in diffs])
    assert d.max() <= 1 and (d == 0).mean() > 0.99
    # composed: a 1 LSB tie flip in one stage may grow by the next factor (<= 1.4): <= 1 per stage
    dc = np.concatenate([x.ravel() for x in composed])
    assert dc.max() <= 3 and (dc == 0).mean() > 0.99
