"""B200-native SAND per-batch view materialisation (Python binding over libsand.so).

Thin marshalling over the C-ABI in ``include/sand.h`` (names match the C
functions). torch supplies device memory, streams and process groups only; every
step of the path runs in libsand.so's CUDA kernels. There is no CPU fallback:
constructing a ``Store`` without the library or a CUDA device raises.

    store = Store(device=0, capacity_bytes=...)
    store.add_video(v, n_frames, W, H); store.put_frames(...)   # decoded NV12
    view = View(store, spec)                                       # open()
    outs = view.alloc_outputs()                                    # torch tensors
    view.read_batch(epoch, rank, iteration, outs)                  # read()
    metas = view.get_meta(epoch, rank, iteration)                  # getxattr()
    view.close(); store.close()                                    # close()
"""
from __future__ import annotations

import ctypes

from . import _abi
from ._abi import (BF16, F32, GEOM_RRC, GEOM_SHORTSIDE_CROP, MAX_GROUPS, MAX_T, MAX_VIEWS, U8, SandError,
                   check, lib)
from .configs import Spec, ViewSpec, Workload

__all__ = ["Store", "View", "plan_rank_clips", "plan_clip", "Spec", "ViewSpec", "Workload", "SandError", "lib", "make_spec",
           "U8", "BF16", "F32", "GEOM_RRC", "GEOM_SHORTSIDE_CROP"]

_TORCH_DTYPE = None


def _torch_dtype(d: int):
    import torch
    return {U8: torch.uint8, BF16: torch.bfloat16, F32: torch.float32}[d]


def make_spec(spec: Spec, videos) -> tuple[_abi.sand_view_spec, object]:
    """Marshal a Spec into sand_view_spec. Returns (struct, keepalive video array)."""
    s = _abi.sand_view_spec()
    s.seed = spec.seed
    s.world_size = spec.world_size
    s.batch_size = spec.batch_size
    s.samples_per_video = spec.samples_per_video
    s.drop_last = int(spec.drop_last)
    arr = (ctypes.c_uint32 * len(videos))(*videos)
    s.videos = ctypes.cast(arr, ctypes.POINTER(ctypes.c_uint32))
    s.n_videos = len(videos)
    s.n_views = len(spec.views)
    s.shared_window = int(spec.shared_window)
    s.pool_epochs = int(getattr(spec, "pool_epochs", 1))
    for i, v in enumerate(spec.views):
        o = s.views[i]
        o.clip_len, o.stride, o.pool_offset, o.spatial_group = v.clip_len, v.stride, v.pool_offset, v.spatial_group
        o.geom = v.geom
        o.scale_min, o.scale_max = v.scale
        o.ratio_min, o.ratio_max = v.ratio
        o.short_side, o.out_h, o.out_w = v.short_side, v.out_h, v.out_w
        o.flip_p, o.rot_p, o.rot_max_deg = v.flip_p, v.rot_p, v.rot_max_deg
        o.blur_p, (o.sigma_min, o.sigma_max) = v.blur_p, v.sigma
        o.blur_ksize, o.blur_truncate = v.blur_ksize, v.blur_truncate
        for c in range(3):
            o.mean[c] = v.mean[c]
            o.std[c] = v.std[c]
        o.out_dtype = v.out_dtype
        o.subsample_of = int(getattr(v, "subsample_of", -1))
        o.color_matrix = int(getattr(v, "color_matrix", 0))
        o.jitter_p = float(getattr(v, "jitter_p", 0.0))
        o.brightness = float(getattr(v, "brightness", 0.0))
        o.contrast = float(getattr(v, "contrast", 0.0))
        o.saturation = float(getattr(v, "saturation", 0.0))
    return s, arr


def _stream(stream):
    """cudaStream_t of `stream` (a raw handle, a torch.cuda.Stream, or None = torch's current)."""
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    return getattr(stream, "cuda_stream", stream)


def plan_rank_clips(spec: Spec, videos, epoch: int, rank: int) -> list[int]:
    """Global clip ids of (epoch, rank) in DistributedSampler order (host-only planner)."""
    s, keep = make_spec(spec, list(videos))
    cap = len(videos) * spec.samples_per_video + spec.world_size
    out = (ctypes.c_uint32 * cap)()
    n = ctypes.c_uint32()
    check(lib().sand_plan_rank_clips(ctypes.byref(s), epoch, rank, out, cap, ctypes.byref(n)),
          "sand_plan_rank_clips")
    return list(out[: n.value])


def plan_clip(spec: Spec, videos, epoch: int, clip: int) -> _abi.sand_clip_meta:
    """Plan of one clip (frame indices, crop boxes, augmentation draws), host-only.

    videos: list of (video_id, n_frames, width, height) in dataset order."""
    s, keep = make_spec(spec, [v[0] for v in videos])
    n = len(videos)
    F = (ctypes.c_uint32 * n)(*[v[1] for v in videos])
    W = (ctypes.c_uint32 * n)(*[v[2] for v in videos])
    H = (ctypes.c_uint32 * n)(*[v[3] for v in videos])
    out = _abi.sand_clip_meta()
    check(lib().sand_plan_clip(ctypes.byref(s), F, W, H, epoch, clip, ctypes.byref(out)), "sand_plan_clip")
    return out


class Store:
    """HBM decoded-frame store keyed by (video, frame) (sand_store_*)."""

    def __init__(self, device: int = 0, capacity_bytes: int = 1 << 30):
        self._h = ctypes.c_void_p()
        check(lib().sand_store_create(device, capacity_bytes, ctypes.byref(self._h)), "sand_store_create")
        self.device = device

    @property
    def handle(self):
        return self._h

    def add_video(self, video: int, n_frames: int, width: int, height: int) -> None:
        check(lib().sand_store_add_video(self._h, video, n_frames, width, height), "sand_store_add_video")

    def put_frames(self, video: int, first_frame: int, n_frames: int, y_ptr: int, y_pitch: int,
                   y_frame_stride: int, uv_ptr: int, uv_pitch: int, uv_frame_stride: int,
                   src_on_device: bool, stream: int = 0) -> None:
        check(lib().sand_store_put_frames(self._h, video, first_frame, n_frames, y_ptr, y_pitch, y_frame_stride,
                                          uv_ptr, uv_pitch, uv_frame_stride, int(src_on_device), stream),
              "sand_store_put_frames")

    def put_frame_batch(self, videos, frames, src_ptr: int, frame_stride: int, pitch: int, uv_offset: int,
                        src_on_device: bool, stream: int = 0) -> None:
        """n frames of any videos from one packed buffer (one H2D copy + one scatter kernel)."""
        n = len(videos)
        assert len(frames) == n
        va = (ctypes.c_uint32 * max(n, 1))(*videos)
        fa = (ctypes.c_uint32 * max(n, 1))(*frames)
        check(lib().sand_store_put_frame_batch(self._h, n, ctypes.cast(va, ctypes.c_void_p),
                                               ctypes.cast(fa, ctypes.c_void_p), src_ptr, frame_stride, pitch,
                                               uv_offset, int(src_on_device), stream), "sand_store_put_frame_batch")

    def frame_layout(self, video: int, frame: int) -> _abi.sand_frame_layout:
        out = _abi.sand_frame_layout()
        check(lib().sand_store_frame_layout(self._h, video, frame, ctypes.byref(out)), "sand_store_frame_layout")
        return out

    def mark_present(self, video: int, first_frame: int, n_frames: int) -> None:
        check(lib().sand_store_mark_present(self._h, video, first_frame, n_frames), "sand_store_mark_present")

    def counters(self) -> _abi.sand_counters:
        out = _abi.sand_counters()
        check(lib().sand_store_counters(self._h, ctypes.byref(out)), "sand_store_counters")
        return out

    def frame_counters(self, video: int, first: int, n: int):
        f = (ctypes.c_uint64 * n)()
        u = (ctypes.c_uint64 * n)()
        check(lib().sand_store_frame_counters(self._h, video, first, n, f, u), "sand_store_frame_counters")
        return list(f), list(u)

    def close(self) -> None:
        if self._h:
            check(lib().sand_store_destroy(self._h), "sand_store_destroy")
            self._h = ctypes.c_void_p()


class View:
    """A view group over one clip stream (sand_view_*): open / read / getxattr / close."""

    def __init__(self, store: Store, spec: Spec, videos):
        self.spec = spec
        self.store = store
        self._spec_c, self._keep = make_spec(spec, list(videos))
        self._h = ctypes.c_void_p()
        check(lib().sand_view_create(store.handle, ctypes.byref(self._spec_c), ctypes.byref(self._h)),
              "sand_view_create")
        self._out = _abi.sand_batch_out()   # reused by read_batch: one View per Python thread
        self._out_ref = ctypes.byref(self._out)
        self._read = lib().sand_view_read_batch

    def output_desc(self, k: int) -> _abi.sand_tensor_desc:
        d = _abi.sand_tensor_desc()
        check(lib().sand_view_output_desc(self._h, k, ctypes.byref(d)), "sand_view_output_desc")
        return d

    def alloc_outputs(self, device=None):
        import torch
        outs = []
        for k in range(len(self.spec.views)):
            d = self.output_desc(k)
            outs.append(torch.empty(tuple(d.dims), dtype=_torch_dtype(d.dtype),
                                    device=device if device is not None else f"cuda:{self.store.device}"))
        return outs

    def iterations(self, epoch: int = 0, rank: int = 0) -> int:
        n = ctypes.c_uint64()
        check(lib().sand_view_iterations(self._h, epoch, rank, ctypes.byref(n)), "sand_view_iterations")
        return n.value

    def read_batch(self, epoch: int, rank: int, iteration: int, outs, stream: int | None = None) -> None:
        o = self._out
        o.iteration = iteration
        if stream is None:
            import torch
            stream = torch.cuda.current_stream(self.store.device).cuda_stream
        o.stream = stream
        for k, t in enumerate(outs):
            o.data[k] = t.data_ptr() if hasattr(t, "data_ptr") else int(t)
        rc = self._read(self._h, epoch, rank, self._out_ref)
        if rc:
            check(rc, "sand_view_read_batch")

    def prefetch_epoch(self, epoch: int, rank: int = 0) -> None:
        check(lib().sand_view_prefetch_epoch(self._h, epoch, rank), "sand_view_prefetch_epoch")

    def get_meta(self, epoch: int, rank: int, iteration: int):
        out = (_abi.sand_clip_meta * self.spec.batch_size)()
        check(lib().sand_view_get_meta(self._h, epoch, rank, iteration, out), "sand_view_get_meta")
        return list(out)

    def batch_bytes(self, epoch: int, rank: int, iteration: int) -> _abi.sand_batch_bytes:
        out = _abi.sand_batch_bytes()
        check(lib().sand_view_batch_bytes(self._h, epoch, rank, iteration, ctypes.byref(out)),
              "sand_view_batch_bytes")
        return out

    def batch_bytes_class(self, epoch: int, rank: int, iteration: int, cls: int) -> _abi.sand_batch_bytes:
        out = _abi.sand_batch_bytes()
        check(lib().sand_view_batch_bytes_class(self._h, epoch, rank, iteration, cls, ctypes.byref(out)),
              "sand_view_batch_bytes_class")
        return out

    def set_object_budget(self, nbytes: int) -> None:
        check(lib().sand_view_set_object_budget(self._h, nbytes), "sand_view_set_object_budget")

    def object_stats(self) -> _abi.sand_object_stats:
        out = _abi.sand_object_stats()
        check(lib().sand_view_object_stats(self._h, ctypes.byref(out)), "sand_view_object_stats")
        return out

    def set_prematerialize(self, slots: int) -> None:
        check(lib().sand_view_set_prematerialize(self._h, slots), "sand_view_set_prematerialize")

    def prematerialize(self, epoch: int, rank: int, iteration: int) -> None:
        check(lib().sand_view_prematerialize(self._h, epoch, rank, iteration), "sand_view_prematerialize")

    def acquire_batch(self, epoch: int, rank: int, iteration: int, stream=None):
        """Device pointers of a pre-materialised batch (one per view), valid until release."""
        ptrs = (ctypes.c_void_p * _abi.MAX_VIEWS)()
        check(lib().sand_view_acquire_batch(self._h, epoch, rank, iteration, _stream(stream), ptrs),
              "sand_view_acquire_batch")
        return [ptrs[k] for k in range(len(self.spec.views))]

    def release_batch(self, epoch: int, rank: int, iteration: int, stream=None) -> None:
        check(lib().sand_view_release_batch(self._h, epoch, rank, iteration, _stream(stream)),
              "sand_view_release_batch")

    def set_timing(self, on: bool) -> None:
        check(lib().sand_view_set_timing(self._h, int(bool(on))), "sand_view_set_timing")

    def class_times(self):
        """(milliseconds, launches) per item class since the previous call (0 mild plain,
        1 heavy plain, 2 rotation/blur)."""
        ms = (ctypes.c_double * 3)()
        n = (ctypes.c_uint64 * 3)()
        check(lib().sand_view_class_times(self._h, ms, n), "sand_view_class_times")
        return list(ms), list(n)

    def stats(self) -> _abi.sand_view_stats:
        out = _abi.sand_view_stats()
        check(lib().sand_view_get_stats(self._h, ctypes.byref(out)), "sand_view_get_stats")
        return out

    def close(self) -> None:
        if self._h:
            check(lib().sand_view_destroy(self._h), "sand_view_destroy")
            self._h = ctypes.c_void_p()
