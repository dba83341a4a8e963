"""GPU parity of the round-2 frame-group kernel k_plainw (csrc/k_plainw.cuh) at the shapes its
launcher distinguishes, each a whole batch compared element by element with the oracle
(R#12 / R#17 bit-exact):

  * outputs up to 128 columns (one column pair per lane, NPJ = 1) and up to 256 (NPJ = 2), with
    half rows that leave lanes idle (200 columns: 50 pairs per 64-lane half);
  * heights that end in partial 64-row bands and 16-row tail bands;
  * the three output dtypes and both normalisations (rint bias folded or not, ViewConst::fold);
  * items with two destinations (two views of one spatial group selecting the same frames);
  * items with three destinations, which k_plainw declines (k_plain serves them).
"""
import pytest

from paper_conf_sosp_yelllhkh25_b200 import configs

from test_gpu_parity_r2 import _run

pytestmark = pytest.mark.gpu

V = configs.ViewSpec
K400_NORM = dict(mean=(0.45, 0.45, 0.45), std=(0.225, 0.225, 0.225))


def _w(name, views, batch=4, n_videos=8):
    return configs.Workload(name, configs.Spec(batch_size=batch, views=views), n_videos, 40, 340, 256, name)


@pytest.mark.parametrize("out,dtype,norm", [
    ((128, 96), configs.BF16, {}),               # NPJ = 1, ImageNet normalisation
    ((200, 136), configs.U8, {}),                 # idle lanes in every half row
    ((256, 72), configs.F32, K400_NORM),          # full NPJ = 2 halves, folded rint bias
    ((96, 200), configs.BF16, K400_NORM),         # tall: 64 + 64 + 64 + 8-row bands
])
def test_plainw_shapes(out, dtype, norm):
    w, h = out
    views = [V(clip_len=4, stride=3, out_w=w, out_h=h, out_dtype=dtype, **norm)]
    _run(_w(f"pw_{w}x{h}", views), None, epochs=(0, 1), its=(0, 1))


@pytest.mark.parametrize("n_views", [2, 3])
def test_plainw_destinations(n_views):
    """n views of one spatial group with the same clip law select the same frames: every item
    has n destinations (2: k_plainw with two register destinations; 3: the k_plain fallback)."""
    views = [V(clip_len=6, stride=2, pool_offset=0, spatial_group=0, **K400_NORM) for _ in range(n_views)]
    _run(_w(f"pw_dest{n_views}", views), None, epochs=(0,), its=(0, 1))
