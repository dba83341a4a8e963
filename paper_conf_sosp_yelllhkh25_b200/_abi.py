"""ctypes declarations of include/sand.h (argument marshalling only).

Every function of the C-ABI is exposed under its C name on the object returned
by ``lib()``. The structs mirror sand.h field for field; ``lib()`` refuses to
load a library whose struct sizes differ from these declarations. No compute
happens here: every step of the path runs in libsand.so's kernels.
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
# SAND_LIB selects another in-tree build of the same library (A/B experiments: libsand_*.so)
LIB_PATH = os.path.join(_HERE, os.environ.get("SAND_LIB", "libsand.so"))

MAX_VIEWS = 8
MAX_GROUPS = 8
MAX_T = 64

OK, EINVAL, ENOENT, ENOMEM, ERANGE, ECUDA, EBUSY = 0, -1, -2, -3, -4, -5, -6
U8, BF16, F32 = 0, 1, 2
GEOM_RRC, GEOM_SHORTSIDE_CROP = 0, 1

u32, u64, i32, dbl, vp = ctypes.c_uint32, ctypes.c_uint64, ctypes.c_int32, ctypes.c_double, ctypes.c_void_p


class sand_frame_layout(ctypes.Structure):
    _fields_ = [("y", u64), ("uv", u64), ("pitch", u32), ("width", u32), ("height", u32),
                ("n_frames", u32), ("frame_stride", u64)]


class sand_counters(ctypes.Structure):
    _fields_ = [("videos", u64), ("frames_present", u64), ("bytes_reserved", u64), ("capacity", u64),
                ("fetches", u64), ("uses", u64), ("batches", u64)]


class sand_view_desc(ctypes.Structure):
    _fields_ = [
        ("clip_len", u32), ("stride", u32), ("pool_offset", i32), ("spatial_group", u32), ("geom", i32),
        ("scale_min", dbl), ("scale_max", dbl), ("ratio_min", dbl), ("ratio_max", dbl),
        ("short_side", u32), ("out_h", u32), ("out_w", u32),
        ("flip_p", dbl), ("rot_p", dbl), ("rot_max_deg", dbl),
        ("blur_p", dbl), ("sigma_min", dbl), ("sigma_max", dbl),
        ("blur_ksize", u32), ("blur_truncate", dbl),
        ("mean", dbl * 3), ("std", dbl * 3), ("out_dtype", i32), ("subsample_of", i32), ("color_matrix", i32),
        ("jitter_p", dbl), ("brightness", dbl), ("contrast", dbl), ("saturation", dbl),
    ]


class sand_view_spec(ctypes.Structure):
    _fields_ = [
        ("seed", u64), ("world_size", u32), ("batch_size", u32), ("samples_per_video", u32),
        ("drop_last", i32), ("videos", ctypes.POINTER(u32)), ("n_videos", u32), ("n_views", u32),
        ("shared_window", i32), ("pool_epochs", u32), ("views", sand_view_desc * MAX_VIEWS),
    ]


class sand_tensor_desc(ctypes.Structure):
    _fields_ = [("dims", u32 * 5), ("dtype", i32), ("bytes", u64)]


class sand_batch_out(ctypes.Structure):
    _fields_ = [("iteration", u64), ("stream", vp), ("data", vp * MAX_VIEWS)]


class sand_clip_meta(ctypes.Structure):
    _fields_ = [
        ("clip", u32), ("video", u32), ("sample", u32), ("pool_start", u32),
        ("frames", (u32 * MAX_T) * MAX_VIEWS),
        ("box", (i32 * 4) * MAX_GROUPS),
        ("flip", u32 * MAX_GROUPS), ("rot_on", u32 * MAX_GROUPS), ("blur_on", u32 * MAX_GROUPS),
        ("blur_r", u32 * MAX_GROUPS), ("theta", dbl * MAX_GROUPS), ("sigma", dbl * MAX_GROUPS),
        ("jitter_on", u32 * MAX_GROUPS), ("jitter_order", u32 * MAX_GROUPS), ("jitter_f", (dbl * 3) * MAX_GROUPS),
    ]


class sand_batch_bytes(ctypes.Structure):
    _fields_ = [("src_sectors", u64), ("src_bytes", u64), ("out_bytes", u64), ("fetches", u64), ("uses", u64)]


class sand_view_stats(ctypes.Structure):
    _fields_ = [("batches", u64), ("kernel_launches", u64), ("plans_built", u64), ("work_items", u64),
                ("plan_build_ns", u64), ("plan_wait_ns", u64), ("read_ns", u64),
                ("plan_cpu_ns", u64), ("plan_buffer_wait_ns", u64), ("lock_wait_ns", u64), ("pending_waits", u64)]


class sand_object_stats(ctypes.Structure):
    _fields_ = [("hits", u64), ("fills", u64), ("misses", u64), ("evictions", u64),
                ("objects", u64), ("bytes_used", u64), ("bytes_budget", u64),
                ("decide_ns", u64), ("stage_ns", u64), ("launch_ns", u64)]


P = ctypes.POINTER
SIGNATURES = {
    "sand_store_create": (ctypes.c_int, [ctypes.c_int, u64, P(vp)]),
    "sand_store_add_video": (ctypes.c_int, [vp, u32, u32, u32, u32]),
    "sand_store_put_frames": (ctypes.c_int, [vp, u32, u32, u32, vp, u64, u64, vp, u64, u64, ctypes.c_int, vp]),
    "sand_store_put_frame_batch": (ctypes.c_int, [vp, u32, vp, vp, vp, u64, u64, u64, ctypes.c_int, vp]),
    "sand_store_frame_layout": (ctypes.c_int, [vp, u32, u32, P(sand_frame_layout)]),
    "sand_store_mark_present": (ctypes.c_int, [vp, u32, u32, u32]),
    "sand_store_counters": (ctypes.c_int, [vp, P(sand_counters)]),
    "sand_store_frame_counters": (ctypes.c_int, [vp, u32, u32, u32, P(u64), P(u64)]),
    "sand_store_destroy": (ctypes.c_int, [vp]),
    "sand_view_create": (ctypes.c_int, [vp, P(sand_view_spec), P(vp)]),
    "sand_view_output_desc": (ctypes.c_int, [vp, u32, P(sand_tensor_desc)]),
    "sand_view_iterations": (ctypes.c_int, [vp, u64, u32, P(u64)]),
    "sand_view_read_batch": (ctypes.c_int, [vp, u64, u32, P(sand_batch_out)]),
    "sand_view_prefetch_epoch": (ctypes.c_int, [vp, u64, u32]),
    "sand_view_get_meta": (ctypes.c_int, [vp, u64, u32, u64, P(sand_clip_meta)]),
    "sand_view_batch_bytes": (ctypes.c_int, [vp, u64, u32, u64, P(sand_batch_bytes)]),
    "sand_view_get_stats": (ctypes.c_int, [vp, P(sand_view_stats)]),
    "sand_view_batch_bytes_class": (ctypes.c_int, [vp, u64, u32, u64, u32, P(sand_batch_bytes)]),
    "sand_view_set_timing": (ctypes.c_int, [vp, ctypes.c_int]),
    "sand_view_set_prematerialize": (ctypes.c_int, [vp, u32]),
    "sand_view_set_object_budget": (ctypes.c_int, [vp, u64]),
    "sand_view_object_stats": (ctypes.c_int, [vp, P(sand_object_stats)]),
    "sand_view_prematerialize": (ctypes.c_int, [vp, u64, u32, u64]),
    "sand_view_acquire_batch": (ctypes.c_int, [vp, u64, u32, u64, vp, P(vp)]),
    "sand_view_release_batch": (ctypes.c_int, [vp, u64, u32, u64, vp]),
    "sand_view_class_times": (ctypes.c_int, [vp, P(ctypes.c_double), P(u64)]),
    "sand_view_destroy": (ctypes.c_int, [vp]),
    "sand_last_error": (ctypes.c_char_p, []),
    "sand_version": (ctypes.c_char_p, []),
    "sand_abi_sizes": (ctypes.c_int, [P(u64)]),
    "sand_plan_rank_clips": (ctypes.c_int, [P(sand_view_spec), u64, u32, P(u32), u32, P(u32)]),
    "sand_plan_clip": (ctypes.c_int, [P(sand_view_spec), P(u32), P(u32), P(u32), u64, u32, P(sand_clip_meta)]),
}

STRUCTS = [sand_frame_layout, sand_counters, sand_view_desc, sand_view_spec, sand_tensor_desc,
           sand_batch_out, sand_clip_meta, sand_batch_bytes]

_lib = None


class SandError(RuntimeError):
    def __init__(self, code: int, where: str, msg: str):
        super().__init__(f"{where} failed with {code}: {msg}")
        self.code = code


def lib():
    """Load libsand.so (in-tree). Raises if it is missing: there is no fallback."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is missing: build it with `python native_build.py product`")
        L = ctypes.CDLL(LIB_PATH)
        for name, (res, args) in SIGNATURES.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        sizes = (u64 * 8)()
        L.sand_abi_sizes(sizes)
        for st, n in zip(STRUCTS, sizes):
            if ctypes.sizeof(st) != n:
                raise RuntimeError(f"ABI layout mismatch for {st.__name__}: {ctypes.sizeof(st)} != {n}")
        _lib = L
    return _lib


def check(rc: int, where: str) -> None:
    if rc != OK:
        raise SandError(rc, where, lib().sand_last_error().decode())
