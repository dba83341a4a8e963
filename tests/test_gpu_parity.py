"""GPU parity: the CUDA path through the C-ABI against the oracle (pytest -m gpu).

For every BASELINE.json workload: (1) the plan (clip ids, frame indices, crop
boxes, flip / rotation / blur draws) is compared BIT-EXACTLY through
sand_view_get_meta; (2) materialised outputs are compared element by element
with oracle renders on the same synthetic frames — whole batches on reduced
stores the oracle finishes in seconds, and sampled frames at the full
BASELINE.json store sizes in the launch configuration bench.py times; (3)
invariants the paper fixes (SlowFast slow == fast[::4], world-size invariance,
exactly-once coverage, reuse accounting) and the error paths.
"""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_sosp_yelllhkh25_b200 import configs
import paper_conf_sosp_yelllhkh25_b200 as sand

from helpers import compare, meta_fields, oracle_render, out_numpy, to_oracle, videos_of

pytestmark = pytest.mark.gpu
SEED = 1234


def _setup(workload, n_videos=None, family=synth.UNIFORM, spec=None):
    vids = videos_of(workload, n_videos)
    per_frame = (workload.width + 63) // 64 * 64 * workload.height * 3 // 2 + 256
    cap = len(vids) * workload.n_frames * per_frame + (1 << 20)
    store = sand.Store(0, cap)
    synth.fill_store(store, vids, family, SEED)
    torch.cuda.synchronize()
    spec = spec or workload.spec
    view = sand.View(store, spec, [v[0] for v in vids])
    ospec = to_oracle(spec)
    ods = oracle.make_dataset(vids)
    return store, view, ospec, ods, vids


def _teardown(store, view):
    view.close()
    store.close()


def _check_meta(view, spec, ospec, ods, n, epoch, rank, it):
    got = [meta_fields(spec, m) for m in view.get_meta(epoch, rank, it)]
    ref = [meta_fields(spec, m) for m in oracle.plan_batch(ospec, ods, n, epoch, rank, it)]
    assert got == ref


def _check_outputs(view, spec, ospec, ods, vids, epoch, rank, it, samples=None, family=synth.UNIFORM):
    outs = view.alloc_outputs()
    view.read_batch(epoch, rank, it, outs)
    torch.cuda.synchronize()
    ometas = oracle.plan_batch(ospec, ods, len(vids), epoch, rank, it)
    W, H = vids[0][2], vids[0][3]
    if samples is None:
        samples = [(b, k, t) for b in range(spec.batch_size) for k, v in enumerate(spec.views)
                   for t in range(v.clip_len)]
    stats = []
    for b, k, t in samples:
        ref = oracle_render(ospec, ometas[b], k, t, family, SEED, W, H)
        got = out_numpy(outs[k][b, :, t])
        stats.append(compare(got, ref, spec.views[k].out_dtype))
    # bit-identical by construction (R#20): report exact-match fraction
    exact = float(np.mean([s["exact"] for s in stats]))
    assert exact == 1.0, f"exact-match fraction {exact}"
    return outs


# ------------------------------------------------------------------ tiny (configs[0]): whole batches

@pytest.mark.parametrize("dtype", [configs.U8, configs.BF16, configs.F32])
@pytest.mark.parametrize("family", [synth.UNIFORM, synth.SMOOTH])
def test_tiny_all_epochs_exact(dtype, family):
    w = configs.tiny()
    w.spec.views[0].out_dtype = dtype
    store, view, ospec, ods, vids = _setup(w, family=family)
    try:
        for epoch in range(6):
            _check_meta(view, w.spec, ospec, ods, 1, epoch, 0, 0)
            _check_outputs(view, w.spec, ospec, ods, vids, epoch, 0, 0, family=family)
    finally:
        _teardown(store, view)


# ------------------------------------------------------------------ reduced stores: whole batches

@pytest.mark.parametrize("name,n_videos,clips", [("k400", 40, None), ("slowfast", 20, None), ("ray", 20, 3),
                                                  ("slowfast_linspace", 20, None)])
def test_reduced_store_whole_batch(name, n_videos, clips):
    w = configs.slowfast_linspace() if name == "slowfast_linspace" else configs.get(name)
    store, view, ospec, ods, vids = _setup(w, n_videos)
    try:
        n_it = view.iterations(0, 0)
        assert n_it == oracle.iterations(ospec, n_videos) >= 1
        for it in range(n_it):
            _check_meta(view, w.spec, ospec, ods, n_videos, 0, 0, it)
        samples = None
        if clips is not None:   # whole clips (every view and frame) of the first `clips` batch slots
            samples = [(b, k, t) for b in range(clips) for k, v in enumerate(w.spec.views) for t in range(v.clip_len)]
        _check_outputs(view, w.spec, ospec, ods, vids, 0, 0, 0, samples=samples)
    finally:
        _teardown(store, view)


@pytest.mark.parametrize("dtype", [configs.BF16, configs.U8, configs.F32])
def test_twoview_rotate_blur_sampled_clips(dtype):
    w = configs.twoview()
    w.spec.batch_size = 8
    for v in w.spec.views:
        v.out_dtype = dtype
    store, view, ospec, ods, vids = _setup(w, 24)
    try:
        for it in range(view.iterations(0, 0)):
            _check_meta(view, w.spec, ospec, ods, 24, 1, 0, it)
        metas = oracle.plan_batch(ospec, ods, 24, 1, 0, 0)
        # every stencil kernel path is exercised: rotation only (rotated straight to the output),
        # blur only, rotation then blur, and the plain resample
        combos = {(bool(m.rot_on[g]), bool(m.blur_on[g])) for m in metas for g in range(2)}
        assert combos == {(False, False), (True, False), (False, True), (True, True)}, combos
        samples = [(b, k, t) for b in range(8) for k in range(2) for t in (0, 7, 15)]
        _check_outputs(view, w.spec, ospec, ods, vids, 1, 0, 0, samples=samples)
    finally:
        _teardown(store, view)


# ------------------------------------------------------------------ full BASELINE.json sizes, sampled

@pytest.mark.parametrize("name", ["k400", "slowfast", "twoview", "ray"])
def test_full_size_sampled(name):
    w = configs.get(name)
    store, view, ospec, ods, vids = _setup(w)
    try:
        rng = np.random.default_rng(7)
        n_it = view.iterations(0, 0)
        for it in (0, n_it - 1):
            _check_meta(view, w.spec, ospec, ods, len(vids), 2, 0, it)
        samples = [(int(rng.integers(w.spec.batch_size)), k, int(rng.integers(v.clip_len)))
                   for k, v in enumerate(w.spec.views) for _ in range(6)]
        _check_outputs(view, w.spec, ospec, ods, vids, 2, 0, n_it - 1, samples=samples)
    finally:
        _teardown(store, view)


# ------------------------------------------------------------------ invariants

def test_slowfast_slow_is_fast_every_fourth_frame():
    w = configs.slowfast()
    store, view, ospec, ods, vids = _setup(w, 16)
    try:
        outs = view.alloc_outputs()
        view.read_batch(0, 0, 0, outs)
        torch.cuda.synchronize()
        fast, slow = outs
        assert torch.equal(slow, fast[:, :, ::4])
    finally:
        _teardown(store, view)


def test_world_size_invariance_and_exactly_once():
    w = configs.k400()
    w.spec.batch_size = 4
    store, view1, ospec, ods, vids = _setup(w, 32)
    spec8 = configs.k400().spec
    spec8.batch_size = 4
    spec8.world_size = 8
    view8 = sand.View(store, spec8, [v[0] for v in vids])
    try:
        by_clip = {}
        for it in range(view1.iterations(0, 0)):
            outs = view1.alloc_outputs()
            view1.read_batch(0, 0, it, outs)
            for b, m in enumerate(view1.get_meta(0, 0, it)):
                by_clip[m.clip] = outs[0][b].clone()
        assert sorted(by_clip) == list(range(32))        # P:L285 exactly once per epoch
        seen = []
        for r in range(8):
            for it in range(view8.iterations(0, r)):
                outs = view8.alloc_outputs()
                view8.read_batch(0, r, it, outs)
                for b, m in enumerate(view8.get_meta(0, r, it)):
                    assert torch.equal(outs[0][b], by_clip[m.clip])
                    seen.append(m.clip)
        assert sorted(seen) == list(range(32))
    finally:
        view8.close()
        _teardown(store, view1)


def test_reuse_accounting_and_batch_bytes_match_oracle():
    w = configs.slowfast()
    store, view, ospec, ods, vids = _setup(w, 16)
    try:
        outs = view.alloc_outputs()
        view.read_batch(0, 0, 0, outs)
        torch.cuda.synchronize()
        bb = view.batch_bytes(0, 0, 0)
        ob = oracle.batch_bytes(ospec, ods, 16, 0, 0, 0)
        assert (bb.src_sectors, bb.out_bytes, bb.fetches, bb.uses) == \
            (ob.src_sectors, ob.out_bytes, ob.fetches, ob.uses)
        c = store.counters()
        assert (c.fetches, c.uses, c.batches) == (ob.fetches, ob.uses, 1)
    finally:
        _teardown(store, view)
    for name in ("k400", "ray", "twoview"):
        w = configs.get(name)
        store, view, ospec, ods, vids = _setup(w, 16 if name == "ray" else 70)
        try:
            bb = view.batch_bytes(0, 0, 0)
            ob = oracle.batch_bytes(ospec, ods, len(vids), 0, 0, 0)
            assert (bb.src_sectors, bb.out_bytes, bb.fetches, bb.uses) == \
                (ob.src_sectors, ob.out_bytes, ob.fetches, ob.uses), name
        finally:
            _teardown(store, view)


# ------------------------------------------------------------------ error paths

def test_error_paths():
    w = configs.tiny()
    vids = videos_of(w)
    store = sand.Store(0, 1 << 24)
    store.add_video(vids[0][0], 16, 64, 64)      # reserved but no frame put yet
    view = sand.View(store, w.spec, [vids[0][0]])
    try:
        outs = view.alloc_outputs()
        with pytest.raises(sand.SandError) as e:
            view.read_batch(0, 0, 0, outs)
        assert e.value.code == sand._abi.ENOENT
        synth.fill_store(store, vids, synth.UNIFORM, SEED)
        view.read_batch(0, 0, 0, outs)
        with pytest.raises(sand.SandError) as e:
            view.read_batch(0, 0, 1, outs)
        assert e.value.code == sand._abi.ERANGE
        with pytest.raises(sand.SandError) as e:
            view.read_batch(0, 0, 0, [outs[0].view(-1)[1:].data_ptr()])
        assert e.value.code == sand._abi.EINVAL
        with pytest.raises(sand.SandError) as e:
            store.close()
        assert e.value.code == sand._abi.EBUSY
        bad = configs.tiny().spec
        bad.views[0].blur_ksize = 4
        with pytest.raises(sand.SandError):
            sand.View(store, bad, [vids[0][0]])
        with pytest.raises(sand.SandError) as e:
            sand.View(store, w.spec, [999999])
        assert e.value.code == sand._abi.ERANGE
    finally:
        view.close()
        store.close()


# ------------------------------------------------------------------ batch put (decoder-output path)

def test_batch_put_matches_per_frame_fill():
    """sand_store_put_frame_batch (one H2D copy + scatter kernel) stores the same bytes as the
    per-frame path: the batch read from a store filled frame batch by frame batch is
    bit-identical to the one read from a store filled by the device generator."""
    w = configs.k400()
    n_videos = 8
    w.spec.batch_size = 4
    vids = videos_of(w, n_videos)
    store_a, view_a, ospec, ods, _ = _setup(w, n_videos)
    W, H, F = w.width, w.height, w.n_frames
    fb = W * H * 3 // 2
    per_frame = (W + 63) // 64 * 64 * H * 3 // 2 + 256
    store_b = sand.Store(0, len(vids) * F * per_frame + (1 << 20))
    try:
        for v in vids:
            store_b.add_video(v[0], F, W, H)
        chunk = 100                              # several calls: the staging buffer is reused
        for v in vids:
            for f0 in range(0, F, chunk):
                n = min(chunk, F - f0)
                y, uv = synth.frames(synth.UNIFORM, SEED, v[0], f0, n, W, H)
                host = torch.empty((n, fb), dtype=torch.uint8).pin_memory()
                hv = host.numpy()
                hv[:, : W * H] = y.reshape(n, -1)
                hv[:, W * H:] = uv.reshape(n, -1)
                # frames given in reverse order: the scatter follows the (video, frame) lists
                order = list(range(n))[::-1]
                packed = torch.stack([host[i] for i in order]).pin_memory()
                store_b.put_frame_batch([v[0]] * n, [f0 + i for i in order], packed.data_ptr(), fb, W, W * H,
                                        False, torch.cuda.current_stream().cuda_stream)
                torch.cuda.synchronize()
        assert store_b.counters().frames_present == n_videos * F
        view_b = sand.View(store_b, w.spec, [v[0] for v in vids])
        try:
            for it in range(view_a.iterations(0, 0)):
                oa, ob = view_a.alloc_outputs(), view_b.alloc_outputs()
                view_a.read_batch(0, 0, it, oa)
                view_b.read_batch(0, 0, it, ob)
                torch.cuda.synchronize()
                for x, y2 in zip(oa, ob):
                    assert torch.equal(x.view(torch.int16), y2.view(torch.int16))
        finally:
            view_b.close()
    finally:
        _teardown(store_a, view_a)
        store_b.close()


def test_batch_put_rejects_unknown_frames():
    store = sand.Store(0, 1 << 24)
    try:
        store.add_video(5, 4, 64, 64)
        buf = torch.zeros(64 * 64 * 3 // 2 * 2, dtype=torch.uint8, device="cuda")
        with pytest.raises(sand.SandError):
            store.put_frame_batch([5, 5], [0, 4], buf.data_ptr(), 64 * 96, 64, 64 * 64, True)
        assert store.counters().frames_present == 0      # nothing copied on error
        store.put_frame_batch([5, 5], [0, 3], buf.data_ptr(), 64 * 96, 64, 64 * 64, True)
        torch.cuda.synchronize()
        assert store.counters().frames_present == 2
    finally:
        store.close()


# ------------------------------------------------------------------ ragged shapes / generic kernel paths

@pytest.mark.parametrize("case", ["stencil_odd", "mixed_dtypes", "heavy_downscale", "blur_max_radius"])
def test_ragged_shapes_whole_batch(case):
    """Shapes off the bench's fast paths: odd output widths (no pair stores, per-byte blur
    windows), mixed dtypes across views (the generic instantiation), heavy down-scaling of a
    small source (the direct-gather kernel at odd sizes), and the largest blur radius (k = 23,
    sigma = 2.9 -> r = 11) with rotation. Whole batches against the oracle."""
    V = configs.ViewSpec
    if case == "stencil_odd":
        views = [V(clip_len=4, stride=3, out_h=29, out_w=37, rot_p=1.0, rot_max_deg=15.0, blur_p=0.5),
                 V(clip_len=4, stride=3, out_h=29, out_w=37, spatial_group=1, blur_p=1.0, flip_p=1.0)]
        src = (98, 70)
    elif case == "mixed_dtypes":
        views = [V(clip_len=6, stride=2, out_h=40, out_w=44, out_dtype=configs.U8, rot_p=0.5, rot_max_deg=10.0),
                 V(clip_len=3, stride=4, out_h=40, out_w=44, spatial_group=1, out_dtype=configs.F32, blur_p=0.5)]
        src = (120, 96)
    elif case == "heavy_downscale":
        views = [V(clip_len=5, stride=2, out_h=21, out_w=23, scale=(0.5, 1.0)),
                 V(clip_len=5, stride=2, out_h=21, out_w=23, spatial_group=1, scale=(0.3, 1.0), out_dtype=configs.F32)]
        src = (640, 360)
    else:
        views = [V(clip_len=4, stride=2, out_h=64, out_w=64, rot_p=1.0, rot_max_deg=10.0, blur_p=1.0,
                   sigma=(2.9, 2.9))]
        src = (160, 128)
    w = configs.Workload(case, configs.Spec(batch_size=3, shared_window=(case == "heavy_downscale"), views=views),
                         6, 24, src[0], src[1], case)
    store, view, ospec, ods, vids = _setup(w)
    try:
        for epoch in (0, 5):
            _check_meta(view, w.spec, ospec, ods, len(vids), epoch, 0, 0)
            _check_outputs(view, w.spec, ospec, ods, vids, epoch, 0, 0)
    finally:
        _teardown(store, view)
