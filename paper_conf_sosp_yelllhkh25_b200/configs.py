"""View specs and store recipes of the five BASELINE.json workloads.

Pure data (no compute). ``Spec``/``ViewSpec`` mirror ``sand_view_spec`` /
``sand_view_desc``; ``Workload`` adds the synthetic store recipe (videos, frame
count, frame size). Field values follow the readings R#10, R#16, R#17, R#23, R#24.
"""
from __future__ import annotations

from dataclasses import dataclass, field, replace

U8, BF16, F32 = 0, 1, 2
BT601, BT709 = 0, 1
GEOM_RRC, GEOM_SHORTSIDE_CROP = 0, 1

KINETICS_MEAN, KINETICS_STD = (0.45, 0.45, 0.45), (0.225, 0.225, 0.225)
IMAGENET_MEAN, IMAGENET_STD = (0.485, 0.456, 0.406), (0.229, 0.224, 0.225)


@dataclass
class ViewSpec:
    clip_len: int = 16
    stride: int = 4
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
    mean: tuple = IMAGENET_MEAN
    std: tuple = IMAGENET_STD
    out_dtype: int = BF16
    subsample_of: int = -1        # >= 0: linspace sub-sample of that view's frames (f4, R#26)
    color_matrix: int = BT601     # YUV -> RGB matrix: BT601 (R#11) or BT709 (f4, R#29)
    jitter_p: float = 0.0         # colour jitter gate (f4, R#30) and torchvision ColorJitter magnitudes
    brightness: float = 0.0
    contrast: float = 0.0
    saturation: float = 0.0


@dataclass
class Spec:
    seed: int = 0
    world_size: int = 1
    batch_size: int = 32
    samples_per_video: int = 1
    drop_last: bool = False
    shared_window: bool = False
    pool_epochs: int = 1          # k-epoch shared frame pool
    views: list = field(default_factory=lambda: [ViewSpec()])


@dataclass
class Workload:
    name: str
    spec: Spec
    n_videos: int
    n_frames: int
    width: int
    height: int
    description: str = ""

    @property
    def frame_bytes(self) -> int:
        return self.width * self.height * 3 // 2

    def with_videos(self, n_videos: int) -> "Workload":
        return replace(self, n_videos=n_videos)


def tiny() -> Workload:
    v = ViewSpec(clip_len=8, stride=2, out_h=32, out_w=32, flip_p=0.5)
    return Workload("tiny", Spec(batch_size=1, views=[v]), 1, 16, 64, 64,
                    "1 video x 16 frames 64x64, one 8-frame clip stride 2, RRC 32x32, flip, ImageNet norm, B=1")


def k400() -> Workload:
    v = ViewSpec(clip_len=16, stride=4, mean=KINETICS_MEAN, std=KINETICS_STD)
    return Workload("k400", Spec(batch_size=32, views=[v]), 1024, 300, 340, 256,
                    "Kinetics-400-shaped: 340x256 NV12, T=16 stride 4, RRC 224, flip, norm 0.45/0.225, B=32 bf16")


def slowfast() -> Workload:
    common = dict(geom=GEOM_SHORTSIDE_CROP, short_side=256, pool_offset=0, mean=KINETICS_MEAN, std=KINETICS_STD)
    fast = ViewSpec(clip_len=32, stride=2, **common)
    slow = ViewSpec(clip_len=8, stride=8, **common)
    return Workload("slowfast", Spec(batch_size=16, views=[fast, slow]), 1024, 300, 340, 256,
                    "SlowFast-shaped: fast 32/2 + slow 8/8 of one clip, short side 256 -> crop 224, flip, B=16 bf16")


def slowfast_linspace() -> Workload:
    """SlowFast with PySlowFast's slow pathway: the 8 slow frames are the fast clip's frames at
    torch.linspace(0, 31, 8).long() = {0, 4, 8, 13, 17, 22, 26, 31}."""
    w = slowfast()
    w.name = "slowfast_linspace"
    w.spec.views[1].subsample_of = 0
    w.description = "SlowFast-shaped with the PySlowFast linspace slow pathway"
    return w


def k400_two_samples() -> Workload:
    """Fig. 9's `samples_per_video: 2`: two clips per video per epoch, each with its own
    temporal and spatial draws (global clip id = video * 2 + sample)."""
    w = k400()
    w.name = "k400_two_samples"
    w.spec.samples_per_video = 2
    w.description = "Kinetics-400-shaped with two sampled clips per video per epoch (Fig. 9 samples_per_video: 2)"
    return w


def slowfast_hd() -> Workload:
    """SlowFast on 1280x720 sources: short side 256 gives W' = floor(1280 * 256 / 720) = 455, a
    real down-scaling by 2.81 on both axes (SURVEY §8(c) reading 10's variant)."""
    w = slowfast()
    w.name = "slowfast_hd"
    w.n_videos, w.n_frames, w.width, w.height = 256, 300, 1280, 720
    w.description = "SlowFast-shaped on 1280x720 NV12: short side 256 (W' = 455) -> crop 224, fast 32/2 + slow 8/8"
    return w


def twoview() -> Workload:
    views = [ViewSpec(clip_len=16, stride=4, spatial_group=q, rot_p=0.5, rot_max_deg=10.0, blur_p=0.5)
             for q in range(2)]
    return Workload("twoview", Spec(batch_size=64, views=views), 1024, 300, 340, 256,
                    "two-view contrastive: 2 groups x (RRC 224, flip, rotate p.5 +-10, blur p.5 k23), B=64 bf16")


def ray() -> Workload:
    views = [ViewSpec(clip_len=16, stride=4, spatial_group=q, scale=(s, 1.0))
             for q, s in enumerate((0.08, 0.2, 0.35, 0.5))]
    return Workload("ray", Spec(batch_size=16, shared_window=True, views=views), 128, 150, 1920, 1080,
                    "Ray HP search: 1080p NV12, 4 trials sharing frames, RRC 224 (scale_min .08/.2/.35/.5), "
                    "shared window, flip, B=16 per rank bf16")


WORKLOADS = {"tiny": tiny, "k400": k400, "slowfast": slowfast, "twoview": twoview, "ray": ray,
             "slowfast_hd": slowfast_hd, "slowfast_linspace": slowfast_linspace, "k400_two_samples": k400_two_samples}


def get(name: str) -> Workload:
    return WORKLOADS[name]()
