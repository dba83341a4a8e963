"""Seeded synthetic NV12 input generator ("input recipe").

The only module shared by the oracle harness and the CUDA product path. It holds
none of the method's arithmetic: it decides the bytes of synthetic "decoded"
frames (BASELINE.json north_star: synthetic raw NV12 frames stand in for decoder
output). Host bytes (``frames``) and device bytes (``fill_device``) are produced
by the same pure byte function in ``nv12_synth.h`` and are bit-identical.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

UNIFORM = 0
SMOOTH = 1

_HERE = os.path.dirname(os.path.abspath(__file__))
_host = None
_cuda = None


def _load_host():
    global _host
    if _host is None:
        path = os.path.join(_HERE, "libsynth_host.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
        lib = ctypes.CDLL(path)
        lib.synth_fill_frames.restype = ctypes.c_int
        lib.synth_fill_frames.argtypes = [
            ctypes.c_int, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32,
            ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p,
            ctypes.c_size_t, ctypes.c_size_t]
        _host = lib
    return _host


def _load_cuda():
    global _cuda
    if _cuda is None:
        path = os.path.join(_HERE, "libsynth_cuda.so")
        if not os.path.exists(path):
            raise RuntimeError(f"{path} missing: run the build first")
        lib = ctypes.CDLL(path)
        lib.synth_fill_frames_cuda.restype = ctypes.c_int
        lib.synth_fill_frames_cuda.argtypes = [
            ctypes.c_int, ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint32, ctypes.c_uint32,
            ctypes.c_uint32, ctypes.c_uint32, ctypes.c_void_p, ctypes.c_size_t, ctypes.c_void_p,
            ctypes.c_size_t, ctypes.c_size_t, ctypes.c_void_p]
        _cuda = lib
    return _cuda


def frames(family: int, seed: int, video: int, first_frame: int, n_frames: int,
           width: int, height: int):
    """Host NV12 frames: returns (y [n,H,W] u8, uv [n,H/2,W] u8), contiguous."""
    if width % 2 or height % 2:
        raise ValueError("NV12 needs even width and height")
    y = np.empty((n_frames, height, width), np.uint8)
    uv = np.empty((n_frames, height // 2, width), np.uint8)
    lib = _load_host()
    # y and uv are separate buffers with different per-frame strides: fill frame by frame
    for f in range(n_frames):
        rc = lib.synth_fill_frames(family, seed, video, first_frame + f, 1, width, height,
                                   y[f].ctypes.data, width, uv[f].ctypes.data, width, 0)
        if rc != 0:
            raise RuntimeError("synth_fill_frames failed")
    return y, uv


def fill_device(family: int, seed: int, video: int, first_frame: int, n_frames: int,
                width: int, height: int, y_ptr: int, y_pitch: int, uv_ptr: int, uv_pitch: int,
                frame_stride: int, stream: int = 0) -> None:
    """Device NV12 frames written in place (pointers are device addresses)."""
    lib = _load_cuda()
    rc = lib.synth_fill_frames_cuda(family, seed, video, first_frame, n_frames, width, height,
                                    y_ptr, y_pitch, uv_ptr, uv_pitch, frame_stride, stream)
    if rc != 0:
        raise RuntimeError(f"synth_fill_frames_cuda failed ({rc})")


def fill_store(store, videos, family: int, seed: int, stream: int = 0) -> None:
    """Write synthetic frames straight into a product frame store (zero-copy).

    ``store`` is a paper_conf_sosp_yelllhkh25_b200.Store; ``videos`` is a list of
    (video_id, n_frames, width, height). Uses only the store's public layout query
    (sand_store_frame_layout) and mark_present; the bytes come from this module.
    """
    for vid, F, W, H in videos:
        store.add_video(vid, F, W, H)
        lay = store.frame_layout(vid, 0)
        fill_device(family, seed, vid, 0, F, W, H, lay.y, lay.pitch, lay.uv, lay.pitch, lay.frame_stride, stream)
        store.mark_present(vid, 0, F)
