"""CPU oracle for SAND's per-batch view materialisation (ctypes wrapper).

TEST INFRASTRUCTURE ONLY: only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import this
package. The product package never imports it.

The arithmetic lives in ``sand_oracle.c`` (plain single-threaded C, every
function citing the PAPER.md passage or DESIGN.md reading it follows). This
module only marshals arguments and declares the C structs again in ctypes.
"""
from __future__ import annotations

import ctypes
import os
from dataclasses import dataclass, field
from typing import Sequence

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
MAX_VIEWS = 8
MAX_GROUPS = 8
MAX_T = 64

U8, BF16, F32 = 0, 1, 2
GEOM_RRC, GEOM_SHORTSIDE_CROP = 0, 1


class View(ctypes.Structure):
    _fields_ = [
        ("clip_len", ctypes.c_uint32), ("stride", ctypes.c_uint32),
        ("pool_offset", ctypes.c_int32), ("spatial_group", ctypes.c_uint32),
        ("geom", ctypes.c_int32),
        ("scale_min", ctypes.c_double), ("scale_max", ctypes.c_double),
        ("ratio_min", ctypes.c_double), ("ratio_max", ctypes.c_double),
        ("short_side", ctypes.c_uint32), ("out_h", ctypes.c_uint32), ("out_w", ctypes.c_uint32),
        ("flip_p", ctypes.c_double), ("rot_p", ctypes.c_double), ("rot_max_deg", ctypes.c_double),
        ("blur_p", ctypes.c_double), ("sigma_min", ctypes.c_double), ("sigma_max", ctypes.c_double),
        ("blur_ksize", ctypes.c_uint32), ("blur_truncate", ctypes.c_double),
        ("mean", ctypes.c_double * 3), ("std", ctypes.c_double * 3),
        ("out_dtype", ctypes.c_int32), ("subsample_of", ctypes.c_int32), ("color_matrix", ctypes.c_int32),
        ("jitter_p", ctypes.c_double), ("brightness", ctypes.c_double), ("contrast", ctypes.c_double),
        ("saturation", ctypes.c_double),
    ]


class Spec(ctypes.Structure):
    _fields_ = [
        ("seed", ctypes.c_uint64), ("world_size", ctypes.c_uint32), ("batch_size", ctypes.c_uint32),
        ("samples_per_video", ctypes.c_uint32), ("drop_last", ctypes.c_int32),
        ("n_views", ctypes.c_uint32), ("shared_window", ctypes.c_int32), ("pool_epochs", ctypes.c_uint32),
        ("views", View * MAX_VIEWS),
    ]


class VideoInfo(ctypes.Structure):
    _fields_ = [("video", ctypes.c_uint32), ("n_frames", ctypes.c_uint32),
                ("width", ctypes.c_uint32), ("height", ctypes.c_uint32)]


class ClipMeta(ctypes.Structure):
    _fields_ = [
        ("clip", ctypes.c_uint32), ("video", ctypes.c_uint32), ("sample", ctypes.c_uint32),
        ("pool_start", ctypes.c_uint32),
        ("frames", (ctypes.c_uint32 * MAX_T) * MAX_VIEWS),
        ("box", (ctypes.c_int32 * 4) * MAX_GROUPS),
        ("flip", ctypes.c_uint32 * MAX_GROUPS), ("rot_on", ctypes.c_uint32 * MAX_GROUPS),
        ("blur_on", ctypes.c_uint32 * MAX_GROUPS), ("blur_r", ctypes.c_uint32 * MAX_GROUPS),
        ("theta", ctypes.c_double * MAX_GROUPS), ("sigma", ctypes.c_double * MAX_GROUPS),
        ("jitter_on", ctypes.c_uint32 * MAX_GROUPS), ("jitter_order", ctypes.c_uint32 * MAX_GROUPS),
        ("jitter_f", (ctypes.c_double * 3) * MAX_GROUPS),
    ]


class FrameRef(ctypes.Structure):
    _fields_ = [("video", ctypes.c_uint32), ("frame", ctypes.c_uint32),
                ("width", ctypes.c_uint32), ("height", ctypes.c_uint32),
                ("y", ctypes.c_void_p), ("uv", ctypes.c_void_p),
                ("y_pitch", ctypes.c_uint64), ("uv_pitch", ctypes.c_uint64)]


class BatchBytes(ctypes.Structure):
    _fields_ = [("src_sectors", ctypes.c_uint64), ("out_bytes", ctypes.c_uint64),
                ("fetches", ctypes.c_uint64), ("uses", ctypes.c_uint64)]


_lib = None


def lib():
    global _lib
    if _lib is None:
        path = os.path.join(_HERE, "libsand_oracle.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `python native_build.py oracle`")
        L = ctypes.CDLL(path)
        P = ctypes.POINTER
        u32, u64, i32, dbl, vp = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int32, ctypes.c_double, ctypes.c_void_p
        sigs = {
            "oracle_philox4x32_10": (None, [P(u32), P(u32), P(u32)]),
            "oracle_u01": (dbl, [u32]),
            "oracle_bounded": (u32, [u32, u32]),
            "oracle_linspace_index": (u32, [u32, u32, u32]),
            "oracle_bern": (ctypes.c_int, [u32, dbl]),
            "oracle_permutation": (None, [u32, u64, u64, P(u32)]),
            "oracle_num_samples": (u32, [u32, u32, ctypes.c_int]),
            "oracle_partition": (u32, [P(u32), u32, u32, u32, ctypes.c_int, P(u32)]),
            "oracle_temporal": (None, [P(Spec), u64, u32, u32, P(ClipMeta)]),
            "oracle_rrc_box": (None, [P(View), u64, u64, u32, u32, u32, u32, P(i32)]),
            "oracle_shortside_box": (None, [P(View), u64, u64, u32, u32, u32, u32, P(i32)]),
            "oracle_spatial": (None, [P(Spec), u64, u32, u32, u32, P(ClipMeta)]),
            "oracle_plan_clip": (None, [P(Spec), P(VideoInfo), u64, u32, P(ClipMeta)]),
            "oracle_iterations": (u64, [P(Spec), u32]),
            "oracle_plan_batch": (ctypes.c_int, [P(Spec), P(VideoInfo), u32, u64, u32, u64, P(ClipMeta)]),
            "oracle_nv12_to_rgb": (None, [vp, ctypes.c_size_t, vp, ctypes.c_size_t, u32, u32, ctypes.c_int, vp]),
            "oracle_resize": (None, [vp, u32, u32, u32, u32, vp]),
            "oracle_resized_crop": (None, [vp, u32, u32, P(i32), u32, u32, vp]),
            "oracle_shortside_crop": (None, [vp, u32, u32, P(i32), u32, u32, vp]),
            "oracle_flip": (None, [vp, u32, u32, vp]),
            "oracle_rotate": (None, [vp, u32, u32, dbl, vp]),
            "oracle_color_jitter": (None, [vp, u32, u32, ctypes.POINTER(ctypes.c_double), u32]),
            "oracle_blur_weights": (None, [dbl, u32, P(ctypes.c_float)]),
            "oracle_blur": (None, [vp, u32, u32, dbl, u32, vp]),
            "oracle_norm_coeffs": (None, [P(dbl), P(dbl), P(ctypes.c_float), P(ctypes.c_float)]),
            "oracle_normalize": (ctypes.c_float, [ctypes.c_uint8, ctypes.c_float, ctypes.c_float]),
            "oracle_bf16_rne": (ctypes.c_uint16, [ctypes.c_float]),
            "oracle_render_frame": (None, [P(Spec), P(ClipMeta), u32, vp, ctypes.c_size_t, vp,
                                           ctypes.c_size_t, u32, u32, vp]),
            "oracle_materialize": (ctypes.c_int, [P(Spec), P(VideoInfo), u32, u64, u32, u64, P(FrameRef),
                                                  u32, P(vp), P(ClipMeta)]),
            "oracle_batch_bytes_of": (ctypes.c_int, [P(Spec), P(VideoInfo), u32, u64, u32, u64, P(BatchBytes)]),
            "oracle_sizeof_spec": (ctypes.c_size_t, []),
            "oracle_sizeof_meta": (ctypes.c_size_t, []),
            "oracle_sizeof_frame_ref": (ctypes.c_size_t, []),
        }
        for name, (res, args) in sigs.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        assert L.oracle_sizeof_spec() == ctypes.sizeof(Spec), "oracle_spec layout mismatch"
        assert L.oracle_sizeof_meta() == ctypes.sizeof(ClipMeta), "oracle_clip_meta layout mismatch"
        assert L.oracle_sizeof_frame_ref() == ctypes.sizeof(FrameRef), "oracle_frame_ref layout mismatch"
        _lib = L
    return _lib


# --------------------------------------------------------------------------- helpers

def _u8p(a: np.ndarray):
    assert a.flags.c_contiguous
    return a.ctypes.data_as(ctypes.c_void_p)


def philox(ctr: Sequence[int], key: Sequence[int]) -> list[int]:
    c = (ctypes.c_uint32 * 4)(*ctr)
    k = (ctypes.c_uint32 * 2)(*key)
    o = (ctypes.c_uint32 * 4)()
    lib().oracle_philox4x32_10(c, k, o)
    return list(o)


def bounded(x: int, n: int) -> int:
    return lib().oracle_bounded(x, n)


def bern(x: int, p: float) -> int:
    return lib().oracle_bern(x, p)


def permutation(n: int, seed: int, epoch: int) -> np.ndarray:
    out = np.empty(max(n, 1), np.uint32)
    lib().oracle_permutation(n, seed, epoch, out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)))
    return out[:n]


def partition(perm: np.ndarray, world: int, rank: int, drop_last: bool) -> np.ndarray:
    perm = np.ascontiguousarray(perm, np.uint32)
    n = len(perm)
    out = np.empty(n // world + 2, np.uint32)
    k = lib().oracle_partition(perm.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)), n, world, rank,
                               int(drop_last), out.ctypes.data_as(ctypes.POINTER(ctypes.c_uint32)))
    return out[:k].copy()


def nv12_to_rgb(y: np.ndarray, uv: np.ndarray, matrix: int = 0) -> np.ndarray:
    """matrix 0: BT.601 (R#11, OpenCV's integer form); 1: BT.709 (R#29)."""
    H, W = y.shape
    y = np.ascontiguousarray(y)
    uv = np.ascontiguousarray(uv)
    out = np.empty((H, W, 3), np.uint8)
    lib().oracle_nv12_to_rgb(_u8p(y), W, _u8p(uv), W, W, H, matrix, _u8p(out))
    return out


def resize(img: np.ndarray, Ho: int, Wo: int) -> np.ndarray:
    img = np.ascontiguousarray(img, np.uint8)
    h, w, _ = img.shape
    out = np.empty((Ho, Wo, 3), np.uint8)
    lib().oracle_resize(_u8p(img), w, h, Ho, Wo, _u8p(out))
    return out


def resized_crop(rgb: np.ndarray, box, Ho: int, Wo: int) -> np.ndarray:
    rgb = np.ascontiguousarray(rgb, np.uint8)
    H, W, _ = rgb.shape
    b = (ctypes.c_int32 * 4)(*box)
    out = np.empty((Ho, Wo, 3), np.uint8)
    lib().oracle_resized_crop(_u8p(rgb), W, H, b, Ho, Wo, _u8p(out))
    return out


def shortside_crop(rgb: np.ndarray, box, Ho: int, Wo: int) -> np.ndarray:
    rgb = np.ascontiguousarray(rgb, np.uint8)
    H, W, _ = rgb.shape
    b = (ctypes.c_int32 * 4)(*box)
    out = np.empty((Ho, Wo, 3), np.uint8)
    lib().oracle_shortside_crop(_u8p(rgb), W, H, b, Ho, Wo, _u8p(out))
    return out


def flip(img: np.ndarray) -> np.ndarray:
    img = np.ascontiguousarray(img, np.uint8)
    Ho, Wo, _ = img.shape
    out = np.empty_like(img)
    lib().oracle_flip(_u8p(img), Ho, Wo, _u8p(out))
    return out


def rotate(img: np.ndarray, theta_deg: float) -> np.ndarray:
    img = np.ascontiguousarray(img, np.uint8)
    Ho, Wo, _ = img.shape
    out = np.empty_like(img)
    lib().oracle_rotate(_u8p(img), Ho, Wo, theta_deg, _u8p(out))
    return out


def color_jitter(img: np.ndarray, factors, order: int) -> np.ndarray:
    """img: HWC uint8; factors (brightness, contrast, saturation); order 0..5 (R#30)."""
    out = np.ascontiguousarray(img, np.uint8).copy()
    H, W, _ = out.shape
    f = (ctypes.c_double * 3)(*factors)
    lib().oracle_color_jitter(_u8p(out), H, W, f, order)
    return out


def blur_weights(sigma: float, r: int) -> np.ndarray:
    w = (ctypes.c_float * 64)()
    lib().oracle_blur_weights(sigma, r, w)
    return np.array(w[: 2 * r + 1], np.float32)


def blur(img: np.ndarray, sigma: float, r: int) -> np.ndarray:
    img = np.ascontiguousarray(img, np.uint8)
    Ho, Wo, _ = img.shape
    out = np.empty_like(img)
    lib().oracle_blur(_u8p(img), Ho, Wo, sigma, r, _u8p(out))
    return out


def norm_coeffs(mean, std):
    m = (ctypes.c_double * 3)(*mean)
    s = (ctypes.c_double * 3)(*std)
    a = (ctypes.c_float * 3)()
    b = (ctypes.c_float * 3)()
    lib().oracle_norm_coeffs(m, s, a, b)
    return np.array(a[:], np.float32), np.array(b[:], np.float32)


def normalize(q: np.ndarray, mean, std, dtype: int) -> np.ndarray:
    """q: HWC u8 -> CHW in dtype (elementwise oracle_normalize / oracle_bf16_rne)."""
    a, b = norm_coeffs(mean, std)
    L = lib()
    H, W, _ = q.shape
    if dtype == U8:
        return np.ascontiguousarray(q.transpose(2, 0, 1))
    out = np.empty((3, H, W), np.float32 if dtype == F32 else np.uint16)
    for c in range(3):
        for y in range(H):
            for x in range(W):
                v = L.oracle_normalize(int(q[y, x, c]), float(a[c]), float(b[c]))
                out[c, y, x] = v if dtype == F32 else L.oracle_bf16_rne(v)
    return out


# --------------------------------------------------------------------------- spec helpers

@dataclass
class ViewDesc:
    clip_len: int = 8
    stride: int = 2
    pool_offset: int = -1
    spatial_group: int = 0
    geom: int = GEOM_RRC
    scale: tuple = (0.08, 1.0)
    ratio: tuple = (3.0 / 4.0, 4.0 / 3.0)
    short_side: int = 0
    out_h: int = 224
    out_w: int = 224
    flip_p: float = 0.5
    rot_p: float = 0.0
    rot_max_deg: float = 0.0
    blur_p: float = 0.0
    sigma: tuple = (0.1, 2.0)
    blur_ksize: int = 23
    blur_truncate: float = 4.0
    mean: tuple = (0.485, 0.456, 0.406)
    std: tuple = (0.229, 0.224, 0.225)
    out_dtype: int = BF16
    subsample_of: int = -1
    color_matrix: int = 0
    jitter_p: float = 0.0
    brightness: float = 0.0
    contrast: float = 0.0
    saturation: float = 0.0


@dataclass
class SpecDesc:
    seed: int = 0
    world_size: int = 1
    batch_size: int = 1
    samples_per_video: int = 1
    drop_last: bool = False
    shared_window: bool = False
    pool_epochs: int = 1
    views: list = field(default_factory=lambda: [ViewDesc()])


def make_spec(sd: SpecDesc) -> Spec:
    s = Spec()
    s.seed = sd.seed
    s.world_size = sd.world_size
    s.batch_size = sd.batch_size
    s.samples_per_video = sd.samples_per_video
    s.drop_last = int(sd.drop_last)
    s.shared_window = int(sd.shared_window)
    s.pool_epochs = int(sd.pool_epochs)
    s.n_views = len(sd.views)
    for i, v in enumerate(sd.views):
        o = s.views[i]
        o.clip_len, o.stride, o.pool_offset, o.spatial_group = v.clip_len, v.stride, v.pool_offset, v.spatial_group
        o.geom = v.geom
        o.scale_min, o.scale_max = v.scale
        o.ratio_min, o.ratio_max = v.ratio
        o.short_side, o.out_h, o.out_w = v.short_side, v.out_h, v.out_w
        o.flip_p, o.rot_p, o.rot_max_deg, o.blur_p = v.flip_p, v.rot_p, v.rot_max_deg, v.blur_p
        o.sigma_min, o.sigma_max = v.sigma
        o.blur_ksize, o.blur_truncate = v.blur_ksize, v.blur_truncate
        for c in range(3):
            o.mean[c] = v.mean[c]
            o.std[c] = v.std[c]
        o.out_dtype = v.out_dtype
        o.subsample_of = v.subsample_of
        o.color_matrix = v.color_matrix
        o.jitter_p, o.brightness, o.contrast, o.saturation = v.jitter_p, v.brightness, v.contrast, v.saturation
    return s


def make_dataset(videos):
    """videos: list of (video_id, n_frames, width, height)."""
    arr = (VideoInfo * max(len(videos), 1))()
    for i, (vid, F, W, H) in enumerate(videos):
        arr[i].video, arr[i].n_frames, arr[i].width, arr[i].height = vid, F, W, H
    return arr


def iterations(spec: Spec, n_videos: int) -> int:
    return lib().oracle_iterations(ctypes.byref(spec), n_videos)


def plan_batch(spec: Spec, dataset, n_videos: int, epoch: int, rank: int, iteration: int):
    metas = (ClipMeta * spec.batch_size)()
    rc = lib().oracle_plan_batch(ctypes.byref(spec), dataset, n_videos, epoch, rank, iteration, metas)
    if rc != 0:
        raise IndexError(f"oracle_plan_batch rc={rc}")
    return metas


def render_frame(spec: Spec, meta: ClipMeta, k: int, y: np.ndarray, uv: np.ndarray) -> np.ndarray:
    v = spec.views[k]
    H, W = y.shape
    y = np.ascontiguousarray(y)
    uv = np.ascontiguousarray(uv)
    dt = {U8: np.uint8, BF16: np.uint16, F32: np.float32}[v.out_dtype]
    out = np.empty((3, v.out_h, v.out_w), dt)
    lib().oracle_render_frame(ctypes.byref(spec), ctypes.byref(meta), k, _u8p(y), W, _u8p(uv), W, W, H,
                              out.ctypes.data_as(ctypes.c_void_p))
    return out


def batch_bytes(spec: Spec, dataset, n_videos: int, epoch: int, rank: int, iteration: int) -> BatchBytes:
    r = BatchBytes()
    rc = lib().oracle_batch_bytes_of(ctypes.byref(spec), dataset, n_videos, epoch, rank, iteration,
                                     ctypes.byref(r))
    if rc != 0:
        raise IndexError(f"oracle_batch_bytes_of rc={rc}")
    return r


def materialize(spec: Spec, dataset, n_videos: int, epoch: int, rank: int, iteration: int,
                frame_refs, outs):
    """outs: list of numpy arrays, one per view, [B,3,T,Ho,Wo] in the view dtype."""
    metas = (ClipMeta * spec.batch_size)()
    ptrs = (ctypes.c_void_p * MAX_VIEWS)(*[o.ctypes.data for o in outs])
    rc = lib().oracle_materialize(ctypes.byref(spec), dataset, n_videos, epoch, rank, iteration,
                                  frame_refs, len(frame_refs), ptrs, metas)
    if rc != 0:
        raise RuntimeError(f"oracle_materialize rc={rc}")
    return metas


def meta_to_dict(spec: Spec, m: ClipMeta) -> dict:
    groups = sorted({spec.views[k].spatial_group for k in range(spec.n_views)})
    return {
        "clip": m.clip, "video": m.video, "sample": m.sample, "pool_start": m.pool_start,
        "frames": [list(m.frames[k][: spec.views[k].clip_len]) for k in range(spec.n_views)],
        "box": {q: list(m.box[q]) for q in groups},
        "flip": {q: m.flip[q] for q in groups}, "rot_on": {q: m.rot_on[q] for q in groups},
        "blur_on": {q: m.blur_on[q] for q in groups}, "blur_r": {q: m.blur_r[q] for q in groups},
        "theta": {q: m.theta[q] for q in groups}, "sigma": {q: m.sigma[q] for q in groups},
    }
