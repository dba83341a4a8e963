"""Test-side glue between the product binding and the oracle (tests only).

Maps the product's Spec to the oracle's spec (field by field), builds synthetic
stores, and compares product outputs with oracle renders under the north_star
tolerances: bit-exact indices/boxes; <= 1 LSB uint8; <= 1e-3 bf16; <= 1e-5 fp32
(R#20: both sides take the uint8 decisions in fp32, so the expected
result is bit-identical and the tests also report the exact-match fraction).
"""
from __future__ import annotations

import numpy as np

import oracle
import synth

SEED_FRAMES = 1234


def to_oracle(spec) -> oracle.Spec:
    views = [oracle.ViewDesc(clip_len=v.clip_len, stride=v.stride, pool_offset=v.pool_offset,
                             spatial_group=v.spatial_group, geom=v.geom, scale=v.scale, ratio=v.ratio,
                             short_side=v.short_side, out_h=v.out_h, out_w=v.out_w, flip_p=v.flip_p,
                             rot_p=v.rot_p, rot_max_deg=v.rot_max_deg, blur_p=v.blur_p, sigma=v.sigma,
                             blur_ksize=v.blur_ksize, blur_truncate=v.blur_truncate, mean=v.mean, std=v.std,
                             out_dtype=v.out_dtype, subsample_of=v.subsample_of,
                             color_matrix=v.color_matrix, jitter_p=v.jitter_p, brightness=v.brightness,
                             contrast=v.contrast, saturation=v.saturation) for v in spec.views]
    return oracle.make_spec(oracle.SpecDesc(seed=spec.seed, world_size=spec.world_size,
                                            batch_size=spec.batch_size, samples_per_video=spec.samples_per_video,
                                            drop_last=spec.drop_last, shared_window=spec.shared_window, pool_epochs=spec.pool_epochs,
                                            views=views))


def videos_of(workload, n_videos=None, first_id=1000):
    n = workload.n_videos if n_videos is None else n_videos
    return [(first_id + i, workload.n_frames, workload.width, workload.height) for i in range(n)]


def meta_fields(spec, m):
    groups = sorted({v.spatial_group for v in spec.views})
    return {
        "clip": m.clip, "video": m.video, "sample": m.sample, "pool_start": m.pool_start,
        "frames": [list(m.frames[k][: v.clip_len]) for k, v in enumerate(spec.views)],
        "box": [list(m.box[q]) for q in groups],
        "flip": [m.flip[q] for q in groups], "rot_on": [m.rot_on[q] for q in groups],
        "blur_on": [m.blur_on[q] for q in groups], "blur_r": [m.blur_r[q] for q in groups],
        "theta": [m.theta[q] for q in groups], "sigma": [m.sigma[q] for q in groups],
        "jitter_on": [m.jitter_on[q] for q in groups], "jitter_order": [m.jitter_order[q] for q in groups],
        "jitter_f": [list(m.jitter_f[q]) for q in groups],
    }


def out_numpy(t):
    """torch output slice -> numpy with the oracle's representation (bf16 as uint16 bits)."""
    import torch
    t = t.detach().cpu().contiguous()
    if t.dtype == torch.bfloat16:
        return t.view(torch.int16).numpy().view(np.uint16)
    return t.numpy()


def bf16_to_f32(bits: np.ndarray) -> np.ndarray:
    return (bits.astype(np.uint32) << 16).view(np.float32)


def compare(got: np.ndarray, ref: np.ndarray, dtype: int) -> dict:
    """North_star tolerances; returns stats and raises AssertionError if violated."""
    if dtype == oracle.U8:
        d = np.abs(got.astype(np.int32) - ref.astype(np.int32))
        assert d.max() <= 1, f"u8 max diff {d.max()}"
    elif dtype == oracle.BF16:
        d = np.abs(bf16_to_f32(got) - bf16_to_f32(ref))
        assert d.max() <= 1e-3, f"bf16 max diff {d.max()}"
    else:
        d = np.abs(got.astype(np.float64) - ref.astype(np.float64))
        assert d.max() <= 1e-5, f"f32 max diff {d.max()}"
    return {"max": float(d.max()), "exact": float((d == 0).mean())}


_frame_cache: dict = {}


def source_frame(family, seed, video, frame, W, H):
    key = (family, seed, video, frame, W, H)
    if key not in _frame_cache:
        if len(_frame_cache) > 4096:
            _frame_cache.clear()
        y, uv = synth.frames(family, seed, video, frame, 1, W, H)
        _frame_cache[key] = (y[0], uv[0])
    return _frame_cache[key]


def oracle_render(ospec, ometa, k, t, family, seed, W, H):
    """Oracle output frame [3, Ho, Wo] of view k, time t of one planned clip."""
    y, uv = source_frame(family, seed, ometa.video, ometa.frames[k][t], W, H)
    return oracle.render_frame(ospec, ometa, k, y, uv)
