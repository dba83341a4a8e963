// planner.cpp — host epoch planner: RNG, permutation, partition, temporal pool,
// spatial draws. Independent of oracle/ (DESIGN.md §4).
#include "planner.h"

#include <algorithm>
#include <cmath>
#include <cstring>
#include <numeric>
#include <string>

#include "plan_types.h"

namespace sand {

// --------------------------------------------------------------------- RNG (R#1)
std::array<uint32_t, 4> Philox4x32::operator()(std::array<uint32_t, 4> x) const {
  constexpr uint64_t kMulA = 0xD2511F53ull, kMulB = 0xCD9E8D57ull;
  constexpr uint32_t kWeylA = 0x9E3779B9u, kWeylB = 0xBB67AE85u;
  uint32_t ka = k0_, kb = k1_;
  for (int r = 0; r < 10; ++r) {
    const uint64_t pa = kMulA * x[0];
    const uint64_t pb = kMulB * x[2];
    x = {static_cast<uint32_t>(pb >> 32) ^ x[1] ^ ka, static_cast<uint32_t>(pb),
         static_cast<uint32_t>(pa >> 32) ^ x[3] ^ kb, static_cast<uint32_t>(pa)};
    ka += kWeylA;
    kb += kWeylB;
  }
  return x;
}

bool draw_coin(uint32_t x, double p) {
  if (!(p > 0.0)) return false;
  if (p >= 1.0) return true;
  return static_cast<uint64_t>(x) < static_cast<uint64_t>(std::floor(p * 4294967296.0));
}

// --------------------------------------------------------------------- spec
static bool same_spatial(const sand_view_desc& a, const sand_view_desc& b) {
  return a.geom == b.geom && a.scale_min == b.scale_min && a.scale_max == b.scale_max &&
         a.ratio_min == b.ratio_min && a.ratio_max == b.ratio_max && a.short_side == b.short_side &&
         a.out_h == b.out_h && a.out_w == b.out_w && a.flip_p == b.flip_p && a.rot_p == b.rot_p &&
         a.rot_max_deg == b.rot_max_deg && a.blur_p == b.blur_p && a.sigma_min == b.sigma_min &&
         a.sigma_max == b.sigma_max && a.blur_ksize == b.blur_ksize && a.blur_truncate == b.blur_truncate &&
         a.jitter_p == b.jitter_p && a.brightness == b.brightness && a.contrast == b.contrast &&
         a.saturation == b.saturation;
}

int validate_spec(const sand_view_spec& s, std::string* why) {
  auto bad = [&](const char* m) { *why = m; return SAND_EINVAL; };
  if (s.world_size == 0) return bad("world_size must be >= 1");
  if (s.batch_size == 0 || s.batch_size > 65535) return bad("batch_size must be in [1, 65535]");
  if (s.samples_per_video == 0) return bad("samples_per_video must be >= 1");
  if (s.n_views == 0 || s.n_views > SAND_MAX_VIEWS) return bad("n_views must be in [1, 8]");
  if (s.n_videos == 0 || s.videos == nullptr) return bad("empty dataset");
  if (static_cast<uint64_t>(s.n_videos) * s.samples_per_video > 0xffffffffull) return bad("too many clips");
  for (uint32_t k = 0; k < s.n_views; ++k) {
    const sand_view_desc& v = s.views[k];
    if (v.clip_len == 0 || v.clip_len > SAND_MAX_T) return bad("clip_len must be in [1, 64]");
    if (v.stride == 0) return bad("stride must be >= 1");
    if (v.spatial_group >= SAND_MAX_GROUPS) return bad("spatial_group must be < 8");
    if (v.geom != SAND_GEOM_RRC && v.geom != SAND_GEOM_SHORTSIDE_CROP) return bad("unknown geom");
    if (v.out_h == 0 || v.out_w == 0 || v.out_h > 4096 || v.out_w > 4096) return bad("bad output size");
    if (v.out_dtype != SAND_U8 && v.out_dtype != SAND_BF16 && v.out_dtype != SAND_F32) return bad("bad dtype");
    if (v.geom == SAND_GEOM_RRC) {
      if (!(v.scale_min > 0.0) || !(v.scale_max >= v.scale_min)) return bad("bad RRC scale range");
      if (!(v.ratio_min > 0.0) || !(v.ratio_max >= v.ratio_min)) return bad("bad RRC ratio range");
    } else if (v.short_side == 0) {
      return bad("SHORTSIDE_CROP needs short_side");
    }
    if (v.blur_ksize % 2 == 0 || v.blur_ksize > 23) return bad("blur_ksize must be odd and <= 23");
    if (v.blur_p > 0.0 && !(v.sigma_min > 0.0 && v.sigma_max >= v.sigma_min)) return bad("bad sigma range");
    if (v.blur_p > 0.0 && (v.blur_ksize - 1) / 2 >= std::min(v.out_h, v.out_w)) return bad("blur radius >= image");
    if ((v.rot_p > 0.0 || v.blur_p > 0.0) && static_cast<uint64_t>(v.out_h) * v.out_w > 65536)
      return bad("rotation/blur views are limited to out_h*out_w <= 65536");
    for (int c = 0; c < 3; ++c)
      if (!(v.std[c] > 0.0)) return bad("std must be > 0");
    for (uint32_t j = 0; j < k; ++j)
      if (s.views[j].spatial_group == v.spatial_group && !same_spatial(s.views[j], v))
        return bad("views of one spatial_group must share all spatial/augmentation fields");
    if (v.subsample_of >= 0 &&
        (static_cast<uint32_t>(v.subsample_of) >= s.n_views || v.subsample_of == static_cast<int32_t>(k) ||
         s.views[v.subsample_of].subsample_of >= 0))
      return bad("subsample_of must name another view that draws from the pool");
    if (v.color_matrix != SAND_BT601 && v.color_matrix != SAND_BT709) return bad("unknown color_matrix");
    if (!(v.jitter_p >= 0.0 && v.jitter_p <= 1.0) || !(v.brightness >= 0.0) || !(v.contrast >= 0.0) ||
        !(v.saturation >= 0.0))
      return bad("colour jitter: probability in [0, 1], magnitudes >= 0");
    if (v.jitter_p > 0.0 && static_cast<uint64_t>(v.out_h) * v.out_w > 65536)
      return bad("colour-jitter views are limited to out_h*out_w <= 65536");
    if (v.color_matrix != s.views[0].color_matrix) return bad("every view must use the same color_matrix");
  }
  uint32_t g = 0;
  for (uint32_t k = 0; k < s.n_views; ++k)
    if (s.views[k].subsample_of < 0) g = std::gcd(g, s.views[k].stride);
  uint32_t L = 0;
  for (uint32_t k = 0; k < s.n_views; ++k)
    if (s.views[k].subsample_of < 0) L = std::max(L, (s.views[k].clip_len - 1) * (s.views[k].stride / g) + 1);
  for (uint32_t k = 0; k < s.n_views; ++k) {
    const sand_view_desc& v = s.views[k];
    if (v.subsample_of < 0 && v.pool_offset >= 0 &&
        static_cast<uint32_t>(v.pool_offset) + (v.clip_len - 1) * (v.stride / g) + 1 > L)
      return bad("pool_offset + span exceeds the shared pool");
  }
  if (s.shared_window)
    for (uint32_t k = 0; k < s.n_views; ++k)
      if (s.views[k].geom != SAND_GEOM_RRC) return bad("shared_window needs RRC views");
  return SAND_OK;
}

void derive_spec(SpecInfo* info) {
  const sand_view_spec& s = info->spec;
  for (int q = 0; q < SAND_MAX_GROUPS; ++q) info->leader[q] = -1;
  info->groups.clear();
  for (uint32_t k = 0; k < s.n_views; ++k) {
    const uint32_t q = s.views[k].spatial_group;
    if (info->leader[q] < 0) info->leader[q] = static_cast<int>(k);
  }
  for (uint32_t q = 0; q < SAND_MAX_GROUPS; ++q)
    if (info->leader[q] >= 0) info->groups.push_back(q);
  uint32_t g = 0;   // the pool is built from the views that draw from it
  for (uint32_t k = 0; k < s.n_views; ++k)
    if (s.views[k].subsample_of < 0) g = std::gcd(g, s.views[k].stride);
  info->g = g;
  info->pool_len = 0;
  for (uint32_t k = 0; k < s.n_views; ++k) {
    info->span[k] = (s.views[k].clip_len - 1) * (s.views[k].stride / g) + 1;
    if (s.views[k].subsample_of < 0) info->pool_len = std::max(info->pool_len, info->span[k]);
  }
}

// --------------------------------------------------------------------- a1: order
uint32_t samples_per_rank(uint32_t n, uint32_t world, bool drop_last) {
  if (drop_last && n % world != 0) return n < world ? 0u : (n - world) / world + ((n - world) % world != 0);
  return n / world + (n % world != 0);
}

std::vector<uint32_t> rank_clips(const SpecInfo& info, uint64_t epoch, uint32_t rank) {
  const sand_view_spec& s = info.spec;
  const uint32_t n = s.n_videos * s.samples_per_video;
  const EpochDraws draws(s.seed, epoch);
  // Fisher-Yates, last position first (R#2)
  std::vector<uint32_t> order(n);
  std::iota(order.begin(), order.end(), 0u);
  for (uint32_t i = n - 1; i >= 1; --i) {
    const uint32_t j = draw_below(draws.get(Purpose::kPerm, 0, 0, 0, i)[0], i + 1);
    std::swap(order[i], order[j]);
  }
  // DistributedSampler(shuffle=False): wrap-pad (or truncate) to num_samples*W, stride W (R#3)
  const uint32_t per_rank = samples_per_rank(n, s.world_size, s.drop_last != 0);
  std::vector<uint32_t> mine;
  mine.reserve(per_rank);
  for (uint32_t i = 0; i < per_rank; ++i) {
    const uint64_t pos = static_cast<uint64_t>(i) * s.world_size + rank;
    mine.push_back(order[static_cast<size_t>(pos % n)]);
  }
  return mine;
}

// --------------------------------------------------------------------- a3: spatial
namespace {

struct CropSize {
  int32_t w, h;
  uint32_t row_draw, col_draw;  // x[2], x[3] of the accepted attempt
  bool accepted;
};

// torchvision RandomResizedCrop.get_params size search in double (R#8)
CropSize rrc_size(const sand_view_desc& v, const EpochDraws& d, uint32_t clip, uint32_t q, uint32_t W,
                  uint32_t H) {
  const double area = static_cast<double>(W) * static_cast<double>(H);
  const double lo = std::log(v.ratio_min), hi = std::log(v.ratio_max);
  for (uint32_t attempt = 0; attempt < 10; ++attempt) {
    const auto x = d.get(Purpose::kCrop, q, 0, attempt, clip);
    const double target = area * (v.scale_min + (v.scale_max - v.scale_min) * draw_unit(x[0]));
    const double aspect = std::exp(lo + (hi - lo) * draw_unit(x[1]));
    const double w = std::nearbyint(std::sqrt(target * aspect));
    const double h = std::nearbyint(std::sqrt(target / aspect));
    if (w > 0.0 && h > 0.0 && w <= W && h <= H)
      return {static_cast<int32_t>(w), static_cast<int32_t>(h), x[2], x[3], true};
  }
  const double in_ratio = static_cast<double>(W) / static_cast<double>(H);
  CropSize c{static_cast<int32_t>(W), static_cast<int32_t>(H), 0, 0, false};
  if (in_ratio < v.ratio_min)
    c.h = static_cast<int32_t>(std::nearbyint(static_cast<double>(W) / v.ratio_min));
  else if (in_ratio > v.ratio_max)
    c.w = static_cast<int32_t>(std::nearbyint(static_cast<double>(H) * v.ratio_max));
  return c;
}

}  // namespace

void plan_clip(const SpecInfo& info, uint64_t epoch, uint32_t clip, sand_clip_meta* m) {
  const sand_view_spec& s = info.spec;
  std::memset(m, 0, sizeof(*m));
  const uint32_t vi = clip / s.samples_per_video;
  const VideoDims& dim = info.dims[vi];
  const uint32_t W = dim.width, H = dim.height, F = dim.n_frames;
  m->clip = clip;
  m->video = dim.id;
  m->sample = clip % s.samples_per_video;
  const EpochDraws d(s.seed, epoch);

  // a2: shared frame pool (R#4, R#5)
  const uint32_t g = info.g, L = info.pool_len;
  const uint32_t pool_frames = (L - 1) * g + 1;
  // the pool is drawn once per chunk of k = pool_epochs epochs (R#25); the views'
  // offsets inside it stay per epoch
  const uint64_t chunk = s.pool_epochs > 1 ? epoch / s.pool_epochs : epoch;
  const EpochDraws dpool(s.seed, chunk);
  const uint32_t start = draw_below(dpool.get(Purpose::kTemporal, 0, 0, 0, clip)[0],
                                    (F > pool_frames ? F - pool_frames : 0u) + 1u);
  m->pool_start = start;
  for (uint32_t k = 0; k < s.n_views; ++k) {
    const sand_view_desc& v = s.views[k];
    if (v.subsample_of >= 0) continue;   // filled from its parent below
    const uint32_t off = v.pool_offset >= 0
                             ? static_cast<uint32_t>(v.pool_offset)
                             : draw_below(d.get(Purpose::kTemporal, 0, 1 + k, 0, clip)[0], L - info.span[k] + 1);
    const uint32_t step = v.stride / g;
    for (uint32_t t = 0; t < v.clip_len; ++t)
      m->frames[k][t] = std::min(start + (off + t * step) * g, F - 1);
  }
  // PySlowFast slow pathway (f4, R#26): the parent's frames at the exact linspace positions
  // floor(t * (T_p - 1) / (T - 1))
  for (uint32_t k = 0; k < s.n_views; ++k) {
    const sand_view_desc& v = s.views[k];
    if (v.subsample_of < 0) continue;
    const uint32_t tp = s.views[v.subsample_of].clip_len;
    for (uint32_t t = 0; t < v.clip_len; ++t) {
      const uint32_t pos = v.clip_len > 1 ? static_cast<uint32_t>(static_cast<uint64_t>(t) * (tp - 1) / (v.clip_len - 1)) : 0u;
      m->frames[k][t] = m->frames[v.subsample_of][pos];
    }
  }

  // a3: crop boxes
  if (s.shared_window) {  // P:L295 (R#18): sizes, then one window, then sub-offsets
    CropSize sz[SAND_MAX_GROUPS] = {};
    int32_t win_w = 0, win_h = 0;
    for (uint32_t q : info.groups) {
      sz[q] = rrc_size(s.views[info.leader[q]], d, clip, q, W, H);
      win_w = std::max(win_w, sz[q].w);
      win_h = std::max(win_h, sz[q].h);
    }
    const auto wdraw = d.get(Purpose::kWindow, 0, 0, 0, clip);
    const int32_t wy = static_cast<int32_t>(draw_below(wdraw[0], H - static_cast<uint32_t>(win_h) + 1));
    const int32_t wx = static_cast<int32_t>(draw_below(wdraw[1], W - static_cast<uint32_t>(win_w) + 1));
    for (uint32_t q : info.groups) {
      const auto x = d.get(Purpose::kWindow, q, 1, 0, clip);
      m->box[q][0] = wx + static_cast<int32_t>(draw_below(x[1], static_cast<uint32_t>(win_w - sz[q].w) + 1));
      m->box[q][1] = wy + static_cast<int32_t>(draw_below(x[0], static_cast<uint32_t>(win_h - sz[q].h) + 1));
      m->box[q][2] = sz[q].w;
      m->box[q][3] = sz[q].h;
    }
  } else {
    for (uint32_t q : info.groups) {
      const sand_view_desc& v = s.views[info.leader[q]];
      if (v.geom == SAND_GEOM_RRC) {
        const CropSize c = rrc_size(v, d, clip, q, W, H);
        if (c.accepted) {
          m->box[q][0] = static_cast<int32_t>(draw_below(c.col_draw, W - static_cast<uint32_t>(c.w) + 1));
          m->box[q][1] = static_cast<int32_t>(draw_below(c.row_draw, H - static_cast<uint32_t>(c.h) + 1));
        } else {  // central crop
          m->box[q][0] = (static_cast<int32_t>(W) - c.w) / 2;
          m->box[q][1] = (static_cast<int32_t>(H) - c.h) / 2;
        }
        m->box[q][2] = c.w;
        m->box[q][3] = c.h;
      } else {  // short side S, then a uniform crop offset (R#9, R#10)
        const uint32_t S = v.short_side;
        const uint32_t Wp = W <= H ? S : static_cast<uint32_t>(static_cast<uint64_t>(W) * S / H);
        const uint32_t Hp = W <= H ? static_cast<uint32_t>(static_cast<uint64_t>(H) * S / W) : S;
        const auto x = d.get(Purpose::kCrop, q, 0, 0, clip);
        m->box[q][0] = static_cast<int32_t>(draw_below(x[3], Wp - v.out_w + 1));
        m->box[q][1] = static_cast<int32_t>(draw_below(x[2], Hp - v.out_h + 1));
        m->box[q][2] = static_cast<int32_t>(Wp);
        m->box[q][3] = static_cast<int32_t>(Hp);
      }
    }
  }

  // gates: flip / rotation / blur (R#15, R#16, R#19)
  for (uint32_t q : info.groups) {
    const sand_view_desc& v = s.views[info.leader[q]];
    const auto x = d.get(Purpose::kAug, q, 0, 0, clip);
    m->flip[q] = draw_coin(x[0], v.flip_p);
    m->rot_on[q] = draw_coin(x[1], v.rot_p);
    m->theta[q] = (2.0 * draw_unit(x[2]) - 1.0) * v.rot_max_deg;
    m->blur_on[q] = draw_coin(x[3], v.blur_p);
    m->sigma[q] = v.sigma_min + (v.sigma_max - v.sigma_min) * draw_unit(d.get(Purpose::kAug, q, 1, 0, clip)[0]);
    const uint32_t cap = (v.blur_ksize - 1) / 2;
    if (v.blur_truncate > 0.0) {
      const double r = std::floor(v.blur_truncate * m->sigma[q] + 0.5);
      m->blur_r[q] = r < static_cast<double>(cap) ? static_cast<uint32_t>(r) : cap;
    } else {
      m->blur_r[q] = cap;
    }
    // colour jitter (R#30): gate and the three factors, then the order of the three ops
    const auto xj = d.get(Purpose::kAug, q, 2, 0, clip);
    m->jitter_on[q] = draw_coin(xj[0], v.jitter_p);
    const double mags[3] = {v.brightness, v.contrast, v.saturation};
    for (int i = 0; i < 3; ++i) {
      const double lo = mags[i] < 1.0 ? 1.0 - mags[i] : 0.0, hi = 1.0 + mags[i];
      m->jitter_f[q][i] = lo + (hi - lo) * draw_unit(xj[1 + i]);
    }
    m->jitter_order[q] = draw_below(d.get(Purpose::kAug, q, 3, 0, clip)[0], 6);
  }
}

}  // namespace sand
