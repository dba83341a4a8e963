// view.cpp — the view group: spec validation, epoch plans, read / getxattr / close
// (SAND view abstraction §5.1; POSIX API Table 2).
//
// Plans are built per (epoch, rank) on the host — synchronously on first use or
// ahead of time by builder threads (read_batch queues the next epochs at iteration 0,
// sand_view_prefetch_epoch queues any; the plan analogue of the paper's
// pre-materialisation threads) — and uploaded once by the builder on the view's
// upload stream, so a read is a presence check, one event wait and one kernel launch on
// the caller's stream.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cmath>
#include <cstdlib>
#include <cstring>

#include "internal.h"
#include "kernels.h"

namespace sand {
namespace {

constexpr size_t kPlanCache = 5;   // current epoch, kPlanAhead ahead, and the previous one
constexpr size_t kMaxPooled = 8;   // idle plan buffers kept for reuse
constexpr size_t kPrealloc = 6;    // spare plan buffers allocated with the first one
}  // namespace
constexpr uint64_t kPlanAhead = 3;
constexpr uint64_t kInflight = 48;   // batches of one view queued on the GPU at most
namespace {
constexpr double kPi = 3.14159265358979323846;

uint64_t now_ns() {
  return static_cast<uint64_t>(
      std::chrono::duration_cast<std::chrono::nanoseconds>(std::chrono::steady_clock::now().time_since_epoch()).count());
}


GroupParams group_params(const sand_view_desc& d, const sand_clip_meta& m, uint32_t q, uint32_t W, uint32_t H) {
  GroupParams g{};
  const int32_t* box = m.box[q];
  if (d.geom == SAND_GEOM_RRC) {           // crop then resize (torchvision resized_crop)
    g.org_x = box[0];
    g.org_y = box[1];
    g.off_x = g.off_y = 0;
    g.lim_x = box[2];
    g.lim_y = box[3];
    g.sc_x = static_cast<float>(box[2]) / static_cast<float>(d.out_w);
    g.sc_y = static_cast<float>(box[3]) / static_cast<float>(d.out_h);
  } else {                                 // resize the frame to W' x H', then crop
    g.org_x = g.org_y = 0;
    g.off_x = box[0];
    g.off_y = box[1];
    g.lim_x = static_cast<int32_t>(W);
    g.lim_y = static_cast<int32_t>(H);
    g.sc_x = static_cast<float>(W) / static_cast<float>(box[2]);
    g.sc_y = static_cast<float>(H) / static_cast<float>(box[3]);
  }
  g.out_w = static_cast<int32_t>(d.out_w);
  g.out_h = static_cast<int32_t>(d.out_h);
  g.flip = static_cast<int32_t>(m.flip[q]);
  g.rot_on = static_cast<int32_t>(m.rot_on[q]);
  const double rad = m.theta[q] * kPi / 180.0;
  g.rot_c = static_cast<float>(std::cos(rad));
  g.rot_s = static_cast<float>(std::sin(rad));
  g.blur_on = static_cast<int32_t>(m.blur_on[q]);
  g.blur_r = static_cast<int32_t>(m.blur_r[q]);
  if (g.blur_on) {  // normalised Gaussian taps in double, cast once (R#16)
    const int r = g.blur_r;
    const double two_s2 = 2.0 * m.sigma[q] * m.sigma[q];
    double e[kMaxTaps];
    double total = 0.0;
    for (int i = 0; i <= 2 * r; ++i) {
      const double dd = static_cast<double>(i) - static_cast<double>(r);
      e[i] = std::exp(-(dd * dd) / two_s2);
      total += e[i];
    }
    for (int i = 0; i <= 2 * r; ++i) g.blur_w[i] = static_cast<float>(e[i] / total);
  }
  g.jit_on = static_cast<int32_t>(m.jitter_on[q]);
  // order k (the k-th permutation of (brightness 0, contrast 1, saturation 2) in lexicographic
  // order) as the op of step s at bits 4 s
  static const int32_t kOrder[6] = {0x210, 0x120, 0x201, 0x021, 0x102, 0x012};
  g.jit_order = kOrder[m.jitter_order[q] % 6];
  for (int i = 0; i < 3; ++i) {   // factors and blend weights in double, cast once (R#30)
    g.jit_f[i] = static_cast<float>(m.jitter_f[q][i]);
    g.jit_a[i] = static_cast<float>(1.0 - m.jitter_f[q][i]);
  }
  return g;
}

}  // namespace

// object-reuse eligibility (f2, R#27): a group whose leader view is a short-side crop without
// rotation or blur (its items are crops of one deterministic resized frame)
bool obj_eligible_group(const sand_view_spec& s, const SpecInfo& info, uint32_t q) {
  const int lead = info.leader[q];
  if (lead < 0) return false;
  const sand_view_desc& d = s.views[lead];
  return d.geom == SAND_GEOM_SHORTSIDE_CROP && d.rot_p <= 0.0 && d.blur_p <= 0.0;
}

namespace {

// staged column span of a group (16-aligned pixels the kernels copy per source row): from the
// first column's i0 to the last column's i1 (taps are monotone; the same set under flip)
int span16(const GroupParams& g) {
  int lo, hi, d;
  float l;
  tap_ref(g.sc_x, g.off_x, 0, g.lim_x, g.org_x, &lo, &d, &l);
  tap_ref(g.sc_x, g.off_x, g.out_w - 1, g.lim_x, g.org_x, &d, &hi, &l);
  return ((hi + 16) & ~15) - (lo & ~15);
}

int row_tap0(const GroupParams& g, int o) {
  int a, b;
  float l;
  tap_ref(g.sc_y, g.off_y, o, g.lim_y, g.org_y, &a, &b, &l);
  return a;
}
int row_tap1(const GroupParams& g, int o) {
  int a, b;
  float l;
  tap_ref(g.sc_y, g.off_y, o, g.lim_y, g.org_y, &a, &b, &l);
  return b;
}

// source rows a k_plain band [y0, y0 + nr) of a group converts (its cost model)
int plain_band_rows(const GroupParams& g, int y0, int nr) { return row_tap1(g, y0 + nr - 1) - row_tap0(g, y0) + 1; }

// k_plain tasks of one batch's mild items [0, n) (ordered by clip slot, group, frame): runs of
// one (clip slot, group) in chunks of `fpc` frames x bands of kPlainRB rows; the costliest first
// (the block scheduler then approximates longest-processing-time order), and the cheapest
// quarter of the work split into kPlainRBTail-row bands so the grid's last wave is short.
// Also returns the widest staged span and the longest band over the tasks.
void plain_tasks(const std::vector<WorkItem>& items, size_t first, size_t n, const std::vector<GroupParams>& groups,
                 int fpc, std::vector<uint2>* out, BatchShape* shape) {
  struct T {
    uint32_t item, nfr, y0, nr;
    double cost;
  };
  std::vector<T> ts;
  auto cost_of = [&](const GroupParams& g, uint32_t nfr, int y0, int nr) {
    const int conv = plain_band_rows(g, y0, nr);
    // lane instructions: ~4.4 per converted channel value, ~8 per output value
    return (double)nfr * (4.4 * 3.0 * conv * span16(g) + 8.0 * 3.0 * nr * g.out_w);
  };
  for (size_t i = 0; i < n;) {
    size_t j = i;
    while (j < n && items[first + j].clip_slot == items[first + i].clip_slot &&
           items[first + j].group == items[first + i].group)
      ++j;
    const GroupParams& g = groups[items[first + i].gp];
    for (size_t f0 = i; f0 < j; f0 += fpc) {
      const uint32_t nfr = (uint32_t)std::min<size_t>(fpc, j - f0);
      for (int y0 = 0; y0 < g.out_h; y0 += kPlainRB) {
        const int nr = std::min(kPlainRB, g.out_h - y0);
        ts.push_back({(uint32_t)f0, nfr, (uint32_t)y0, (uint32_t)nr, cost_of(g, nfr, y0, nr)});
      }
    }
    i = j;
  }
  std::stable_sort(ts.begin(), ts.end(), [](const T& a, const T& b) { return a.cost > b.cost; });
  double total = 0.0;
  for (const T& t : ts) total += t.cost;
  std::vector<T> big, tail;
  double acc = 0.0;
  for (auto it = ts.rbegin(); it != ts.rend(); ++it) {   // cheapest first
    acc += it->cost;
    if (acc <= kPlainTailFrac * total && (int)it->nr > kPlainRBTail) {
      const GroupParams& g = groups[items[first + it->item].gp];
      for (uint32_t y = it->y0; y < it->y0 + it->nr; y += kPlainRBTail) {
        const uint32_t nr = std::min<uint32_t>(kPlainRBTail, it->y0 + it->nr - y);
        tail.push_back({it->item, it->nfr, y, nr, cost_of(g, it->nfr, (int)y, (int)nr)});
      }
    } else {
      big.push_back(*it);
    }
  }
  std::reverse(big.begin(), big.end());
  std::stable_sort(tail.begin(), tail.end(), [](const T& a, const T& b) { return a.cost > b.cost; });
  shape->task_first = (uint32_t)out->size();
  shape->pl_gw = shape->pl_rb = shape->pl_gw_w = 0;
  // per task (not per batch maximum): tasks whose span k_plainw can stage first, then the rest
  for (int wide = 0; wide < 2; ++wide)
    for (const auto* v : {&big, &tail})
      for (const T& t : *v) {
        const GroupParams& g = groups[items[first + t.item].gp];
        const int span = span16(g);
        if ((span > kPlainwMaxSpan) != (wide == 1)) continue;
        shape->pl_gw = std::max(shape->pl_gw, span);
        if (!wide) shape->pl_gw_w = std::max(shape->pl_gw_w, span);
        shape->pl_rb = std::max(shape->pl_rb, (int)t.nr);
        out->push_back(make_uint2(t.item, pl_task_y(t.nfr, t.nr, t.y0)));
      }
  shape->n_tasks = (uint32_t)out->size() - shape->task_first;
  shape->n_tasks_w = 0;
  for (uint32_t i = shape->task_first; i < (uint32_t)out->size(); ++i) {
    const WorkItem& w = items[first + (*out)[i].x];
    if (span16(groups[w.gp]) > kPlainwMaxSpan) break;
    shape->n_tasks_w++;
  }
}

}  // namespace

void shape_items(const sand_view& v, std::vector<WorkItem>& items, const std::vector<GroupParams>& groups,
                 const std::vector<uint32_t>& dests, const ViewConst* views, uint32_t n_views, std::vector<uint2>* tasks,
                 BatchShape* shape) {
  BatchShape sh{};
  sh.fold = 1;
  for (uint32_t k = 0; k < n_views; ++k) sh.fold &= views[k].fold;
  sh.direct_identity = 1;
  sh.src_w_mod4 = 1;
  sh.even_wo = sh.wo_mod4 = 1;
  sh.dtype = -2;   // unset
  for (auto& w : items) {
    const GroupParams& g = groups[w.gp];
    const bool mild = g.sc_x <= 2.0f && g.sc_y <= 2.0f;
    const int cols = span16(g);
    w.flags = (g.rot_on || g.blur_on || g.jit_on) ? 1u : (mild ? 0u : 2u);
    for (uint32_t d = 0; d < w.n_dest; ++d) {
      const ViewConst& vc = views[dests[w.dest_begin + d] >> 24];
      sh.dtype = sh.dtype == -2 ? vc.dtype : (sh.dtype == vc.dtype ? sh.dtype : -1);
      if (vc.out_w & 1) sh.even_wo = 0;
      if (vc.out_w & 3) sh.wo_mod4 = 0;
    }
    if (w.flags & 1u) {
      sh.has_stencil = 1;
      if (g.jit_on) sh.has_jitter = 1;
      sh.st_max_wo = std::max(sh.st_max_wo, g.out_w);
      sh.st_max_ho = std::max(sh.st_max_ho, g.out_h);
      sh.st_cols_bound = std::max(sh.st_cols_bound, cols);
      sh.st_max_scy = std::max(sh.st_max_scy, g.sc_y);
    } else {
      sh.has_direct = 1;
      sh.max_dests = std::max<int32_t>(sh.max_dests, static_cast<int32_t>(w.n_dest));
      if (mild) {
        if (!(g.sc_x == 1.0f && g.sc_y == 1.0f)) sh.direct_identity = 0;
        if (w.src_w % 4u) sh.src_w_mod4 = 0;
        sh.max_wo = std::max(sh.max_wo, g.out_w);
        sh.max_ho = std::max(sh.max_ho, g.out_h);
        sh.cols_bound = std::max(sh.cols_bound, cols);
        sh.max_scy = std::max(sh.max_scy, g.sc_y);
      } else {
        sh.heavy_max_wo = std::max(sh.heavy_max_wo, g.out_w);
        sh.heavy_max_ho = std::max(sh.heavy_max_ho, g.out_h);
      }
    }
  }
  if (sh.dtype == -2) sh.dtype = -1;
  auto mid = std::stable_partition(items.begin(), items.end(), [](const WorkItem& w) { return !(w.flags & 1u); });
  sh.n_direct = static_cast<uint32_t>(mid - items.begin());
  auto hv = std::stable_partition(items.begin(), mid, [](const WorkItem& w) { return !(w.flags & 2u); });
  sh.n_mild = static_cast<uint32_t>(hv - items.begin());
  std::stable_sort(items.begin(), hv, [](const WorkItem& a, const WorkItem& b) {
    return a.clip_slot != b.clip_slot ? a.clip_slot < b.clip_slot : a.group < b.group;
  });
  plain_tasks(items, 0, sh.n_mild, groups, v.pl_fpc, tasks, &sh);
  *shape = sh;
}

std::shared_ptr<EpochPlan> build_plan(const sand_view& v, uint64_t epoch, uint32_t rank,
                                      std::shared_ptr<EpochPlan> plan) {
  const SpecInfo& info = v.info;
  const sand_view_spec& s = info.spec;
  const uint32_t B = s.batch_size;
  const uint32_t nG = static_cast<uint32_t>(info.groups.size());
  // a recycled plan keeps its vectors' capacity: no allocation or page faults per epoch
  if (!plan) plan = std::make_shared<EpochPlan>();
  plan->epoch = epoch;
  plan->rank = rank;
  plan->last_touch = 0;
  plan->items.clear();
  plan->dests.clear();
  plan->tasks.clear();
  plan->item_begin.clear();
  plan->shapes.clear();
  plan->fetch_begin.clear();
  plan->fetch_keys.clear();
  plan->fetch_uses.clear();
  plan->fetch_entry.clear();
  const std::vector<uint32_t> clips = rank_clips(info, epoch, rank);
  plan->iterations = clips.size() / B;
  const uint64_t n_clips = plan->iterations * B;
  plan->metas.resize(n_clips);            // every entry is overwritten by plan_clip
  plan->groups.resize(n_clips * nG);      // ... and by group_params
  uint32_t frames_per_clip = 0;
  for (uint32_t k = 0; k < s.n_views; ++k) frames_per_clip += s.views[k].clip_len;
  plan->items.reserve(n_clips * frames_per_clip * nG);
  plan->dests.reserve(n_clips * frames_per_clip);
  plan->item_begin.reserve(plan->iterations + 1);
  plan->fetch_begin.reserve(plan->iterations + 1);
  plan->shapes.reserve(plan->iterations);
  plan->item_begin.push_back(0);
  plan->fetch_begin.push_back(0);
  std::vector<uint64_t> uses_of;   // (frame << 32) | (view << 16) | t
  std::vector<uint64_t> later;     // (epoch delta << 48) | (group << 32) | frame of later epochs (f2)
  uses_of.reserve(frames_per_clip);
  std::vector<uint32_t> batch_videos(B);
  int32_t common_dtype = s.views[0].out_dtype;
  int32_t even_wo = 1, wo_mod4 = 1;
  for (uint32_t k = 0; k < s.n_views; ++k) {
    if (s.views[k].out_dtype != common_dtype) common_dtype = -1;
    if (s.views[k].out_w & 1u) even_wo = 0;
    if (s.views[k].out_w & 3u) wo_mod4 = 0;
  }
  for (uint64_t it = 0; it < plan->iterations; ++it) {
    BatchShape shape{};
    shape.fold = 1;
    for (uint32_t k = 0; k < s.n_views; ++k) shape.fold &= v.vconst[k].fold;
    shape.direct_identity = 1;
    shape.src_w_mod4 = 1;
    shape.dtype = common_dtype;
    shape.even_wo = even_wo;
    shape.wo_mod4 = wo_mod4;
    struct Fetch {
      uint64_t key;   // (video << 32) | frame
      uint32_t uses;
      VideoEntry* entry;
      bool operator<(const Fetch& o) const { return key < o.key; }
    };
    std::vector<Fetch> fetch;
    fetch.reserve(B * frames_per_clip);
    for (uint32_t b = 0; b < B; ++b) {
      const uint64_t slot = it * B + b;
      sand_clip_meta& m = plan->metas[slot];
      const uint32_t clip = clips[slot];
      plan_clip(info, epoch, clip, &m);
      const VideoDims& dim = info.dims[clip / s.samples_per_video];
      // object reuse (f2, R#27): frames this clip selects, per object-eligible group, in the later
      // epochs of the current k-epoch chunk (their count and the next one travel in WorkItem.pad)
      const uint32_t kch = std::max<uint32_t>(1, s.pool_epochs);
      const uint64_t chunk_end = (epoch / kch + 1) * kch;
      later.clear();
      if (v.obj_budget > 0)
        for (uint64_t e2 = epoch + 1; e2 < chunk_end; ++e2) {
          sand_clip_meta m2;
          plan_clip(info, e2, clip, &m2);
          for (uint32_t k = 0; k < s.n_views; ++k)
            if (obj_eligible_group(s, info, s.views[k].spatial_group))
              for (uint32_t t = 0; t < s.views[k].clip_len; ++t)
                later.push_back((static_cast<uint64_t>(e2 - epoch) << 48) |
                                (static_cast<uint64_t>(s.views[k].spatial_group) << 32) | m2.frames[k][t]);
        }
      VideoEntry* ent = v.entries[clip / s.samples_per_video];
      for (uint32_t gi = 0; gi < nG; ++gi) {
        const uint32_t q = info.groups[gi];
        plan->groups[slot * nG + gi] = group_params(s.views[info.leader[q]], m, q, dim.width, dim.height);
      }
      // launch-shape contribution and stencil flag of each group (independent of the frame)
      uint32_t gflags[SAND_MAX_GROUPS];
      for (uint32_t gi = 0; gi < nG; ++gi) {
        const GroupParams& g = plan->groups[slot * nG + gi];
        // the exact staged span (16-aligned; an estimate capped at 2 * out_w let a
        // wide crop overrun the staging kernels' shared memory)
        const int cols = span16(g);
        const bool mild = g.sc_x <= 2.0f && g.sc_y <= 2.0f;
        gflags[gi] = (g.rot_on || g.blur_on || g.jit_on) ? 1u : (mild ? 0u : 2u);
        if (gflags[gi] & 1u) {
          shape.has_stencil = 1;
          if (g.jit_on) shape.has_jitter = 1;
          shape.st_max_wo = std::max(shape.st_max_wo, g.out_w);
          shape.st_max_ho = std::max(shape.st_max_ho, g.out_h);
          shape.st_cols_bound = std::max(shape.st_cols_bound, cols);
          shape.st_max_scy = std::max(shape.st_max_scy, g.sc_y);
        } else if (mild) {
          shape.has_direct = 1;
          if (!(g.sc_x == 1.0f && g.sc_y == 1.0f)) shape.direct_identity = 0;
          if (dim.width % 4u) shape.src_w_mod4 = 0;
          shape.max_wo = std::max(shape.max_wo, g.out_w);
          shape.max_ho = std::max(shape.max_ho, g.out_h);
          shape.cols_bound = std::max(shape.cols_bound, cols);
          shape.max_scy = std::max(shape.max_scy, g.sc_y);
        } else {
          shape.has_direct = 1;
          shape.heavy_max_wo = std::max(shape.heavy_max_wo, g.out_w);
          shape.heavy_max_ho = std::max(shape.heavy_max_ho, g.out_h);
        }
      }
      // (frame, view, t) uses of the clip sorted by frame: one pass groups the destinations of
      // each unique source frame (view-major, t ascending within a frame)
      uses_of.clear();
      for (uint32_t k = 0; k < s.n_views; ++k)
        for (uint32_t t = 0; t < s.views[k].clip_len; ++t)
          uses_of.push_back((static_cast<uint64_t>(m.frames[k][t]) << 32) | (k << 16) | t);
      std::sort(uses_of.begin(), uses_of.end());
      for (size_t i = 0; i < uses_of.size();) {
        const uint32_t f = static_cast<uint32_t>(uses_of[i] >> 32);
        size_t j = i;
        while (j < uses_of.size() && static_cast<uint32_t>(uses_of[j] >> 32) == f) ++j;
        uint32_t uses = 0;
        for (uint32_t gi = 0; gi < nG; ++gi) {
          const uint32_t q = info.groups[gi];
          WorkItem w{};
          w.dest_begin = static_cast<uint32_t>(plan->dests.size());
          for (size_t x = i; x < j; ++x) {
            const uint32_t k = static_cast<uint32_t>(uses_of[x] >> 16) & 0xffffu;
            if (s.views[k].spatial_group == q)
              plan->dests.push_back(pack_dest(k, static_cast<uint32_t>(uses_of[x]) & 0xffffu, b));
          }
          w.n_dest = static_cast<uint32_t>(plan->dests.size()) - w.dest_begin;
          if (w.n_dest == 0) continue;
          if (!(gflags[gi] & 1u)) shape.max_dests = std::max<int32_t>(shape.max_dests, static_cast<int32_t>(w.n_dest));
          uses += w.n_dest;
          w.y_off = ent->offset + ent->frame_stride * f;
          w.pitch = ent->pitch;
          w.src_w = dim.width;
          w.src_h = dim.height;
          w.gp = static_cast<uint32_t>(slot * nG + gi);
          w.clip_slot = b;
          w.group = q;
          w.flags = gflags[gi];
          if (!later.empty() && !(gflags[gi] & 1u) && obj_eligible_group(s, info, q)) {
            uint32_t uses = 0, next = 0xffffu;   // later epochs selecting frame f for group q
            uint64_t last_e = 0;
            for (uint64_t x : later)
              if (((x >> 32) & 0xffffu) == q && static_cast<uint32_t>(x) == f && (x >> 48) != last_e) {
                last_e = x >> 48;
                ++uses;
                next = std::min<uint32_t>(next, static_cast<uint32_t>(last_e));
              }
            w.pad = (uses << 16) | next;
          } else {
            w.pad = 0xffffu;                    // no later use known
          }
          plan->items.push_back(w);
        }
        fetch.push_back({(static_cast<uint64_t>(dim.id) << 32) | f, uses, ent});
        i = j;
      }
      batch_videos[b] = dim.id;
    }
    // batch-unique (video, frame): clips of different videos never share a frame, so merging
    // (sort + run-length) is only needed when a video occurs twice in the batch
    std::sort(batch_videos.begin(), batch_videos.begin() + B);
    const bool shared = std::adjacent_find(batch_videos.begin(), batch_videos.begin() + B) != batch_videos.begin() + B;
    if (shared) std::sort(fetch.begin(), fetch.end());
    for (size_t i = 0; i < fetch.size();) {
      size_t j = i;
      uint32_t uses = 0;
      while (j < fetch.size() && fetch[j].key == fetch[i].key) uses += fetch[j++].uses;
      plan->fetch_keys.push_back({static_cast<uint32_t>(fetch[i].key >> 32), static_cast<uint32_t>(fetch[i].key)});
      plan->fetch_uses.push_back(uses);
      plan->fetch_entry.push_back(fetch[i].entry);
      i = j;
    }
    plan->fetch_begin.push_back(static_cast<uint32_t>(plan->fetch_keys.size()));
    // direct items first, stencil items after (order kept within each class): each kernel
    // then walks a dense slice instead of skipping the other class's items
    {
      auto first = plan->items.begin() + plan->item_begin.back();
      auto mid = std::stable_partition(first, plan->items.end(), [](const sand::WorkItem& w) { return !(w.flags & 1u); });
      shape.n_direct = static_cast<uint32_t>(mid - first);
      // direct items: mild (k_plain) before heavy (k_direct); mild ones in (clip slot, group,
      // frame) order so the frames of one clip group are adjacent (a k_plain task)
      auto hv = std::stable_partition(first, mid, [](const sand::WorkItem& w) { return !(w.flags & 2u); });
      shape.n_mild = static_cast<uint32_t>(hv - first);
      std::stable_sort(first, hv, [](const sand::WorkItem& a, const sand::WorkItem& b) {
        return a.clip_slot != b.clip_slot ? a.clip_slot < b.clip_slot : a.group < b.group;
      });
      plain_tasks(plan->items, static_cast<size_t>(plan->item_begin.back()), shape.n_mild, plan->groups, v.pl_fpc,
                  &plan->tasks, &shape);
      // stencil items longest first (one CTA per item, dispatched in order): the grid's last
      // wave then holds the cheapest items. Cost model in lane instructions per output value
      // (ncu): resample ~15, rotation ~28, blur ~10 + 3 r.
      auto cost = [&](const sand::WorkItem& w) {
        const sand::GroupParams& g = plan->groups[w.gp];
        return 15 + (g.rot_on ? 28 : 0) + (g.blur_on ? 10 + 3 * g.blur_r : 0);
      };
      std::stable_sort(mid, plan->items.end(),
                       [&](const sand::WorkItem& a, const sand::WorkItem& b) { return cost(a) > cost(b); });
    }
    plan->item_begin.push_back(static_cast<uint32_t>(plan->items.size()));
    plan->shapes.push_back(shape);
  }
  return plan;
}

namespace {

// return a plan's buffers to the view's pool (caller holds v->mu). The next owner waits on
// the buffer's events before overwriting it.
void release_plan_device(sand_view* v, EpochPlan& p) {
  if (p.d_buf) {
    PlanBuffer b;
    b.d = p.d_buf;
    b.h = p.h_stage;
    b.bytes = p.d_bytes;
    b.done = p.last_use;
    b.ready = p.ready;
    v->pool.push_back(b);
  }
  p.d_buf = p.h_stage = nullptr;
  p.last_use = p.ready = nullptr;
  p.uploaded = false;
}

void destroy_buffer(PlanBuffer& b) {
  if (b.done) {
    cudaEventSynchronize(b.done);
    cudaEventDestroy(b.done);
  }
  if (b.ready) {
    cudaEventSynchronize(b.ready);
    cudaEventDestroy(b.ready);
  }
  cudaFree(b.d);
  cudaFreeHost(b.h);
}

void free_pool(sand_view* v) {
  for (auto& b : v->pool) destroy_buffer(b);
  v->pool.clear();
}

struct PlanLayout {
  size_t gb, ib, db, tb, off_i, off_d, off_t, total;
};

PlanLayout plan_layout(const EpochPlan& p) {
  PlanLayout L;
  L.gb = p.groups.size() * sizeof(GroupParams);
  L.ib = p.items.size() * sizeof(WorkItem);
  L.db = p.dests.size() * sizeof(uint32_t);
  L.tb = p.tasks.size() * sizeof(uint2);
  L.off_i = (L.gb + 255) / 256 * 256;
  L.off_d = L.off_i + (L.ib + 255) / 256 * 256;
  L.off_t = L.off_d + (L.db + 255) / 256 * 256;
  L.total = std::max<size_t>(L.off_t + L.tb, 256);
  return L;
}

// Caller holds v->mu: the smallest pooled buffer of at least `bytes` whose previous owner's
// kernels and upload have completed, or an empty one (the builder then allocates a new buffer).
// Evicted plans may still have batches queued on the GPU when the host runs ahead; taking
// such a buffer would make the builder wait for the GPU and leave the next epoch's plan late.
PlanBuffer take_buffer(sand_view* v, size_t bytes) {
  int best = -1;
  for (size_t i = 0; i < v->pool.size(); ++i) {
    const PlanBuffer& b = v->pool[i];
    if (b.bytes < bytes || (best >= 0 && b.bytes >= v->pool[best].bytes)) continue;
    if ((b.done && cudaEventQuery(b.done) != cudaSuccess) || (b.ready && cudaEventQuery(b.ready) != cudaSuccess))
      continue;
    best = (int)i;
  }
  PlanBuffer buf;
  if (best >= 0) {
    buf = v->pool[best];
    v->pool.erase(v->pool.begin() + best);
  } else if (v->pool.size() >= kMaxPooled) {   // bound the pool: wait for the oldest instead
    buf = v->pool.front();
    v->pool.erase(v->pool.begin());
    if (buf.bytes < bytes) {
      destroy_buffer(buf);
      buf = PlanBuffer{};
    }
  }
  return buf;
}

// Allocate a plan buffer of `bytes` (device copy, pinned staging copy, events).
int alloc_buffer(size_t bytes, PlanBuffer* buf) {
  buf->bytes = bytes;
  const char* what = "cudaMalloc(plan)";
  cudaError_t e = cudaMalloc(&buf->d, buf->bytes);
  if (e == cudaSuccess) e = cudaMallocHost(&buf->h, buf->bytes), what = "cudaMallocHost(plan)";
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&buf->done, cudaEventDisableTiming), what = "cudaEventCreate";
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&buf->ready, cudaEventDisableTiming);
  if (e != cudaSuccess) {
    destroy_buffer(*buf);
    *buf = PlanBuffer{};
    return cuda_error(e, what);
  }
  return SAND_OK;
}

// Upload a built plan into buf (allocated here if empty) on the view's upload stream; runs on
// the builder thread without v->mu. On failure the buffer is handed back through *buf.
int upload_plan(sand_view* v, EpochPlan& p, PlanBuffer* buf) {
  const PlanLayout L = plan_layout(p);
  cudaError_t e = cudaSetDevice(v->store->device);
  if (e != cudaSuccess) return cuda_error(e, "cudaSetDevice");
  if (!buf->d) {
    // the first allocation also fills the pool with spares of the same size (+25 %): pinned and
    // device allocations take driver locks and can stall the launching thread, so none happen
    // once batches are being read
    const size_t bytes = L.total + L.total / 4;
    const int rc = alloc_buffer(bytes, buf);
    if (rc != SAND_OK) return rc;
    std::vector<PlanBuffer> spares;
    {
      std::lock_guard<std::mutex> lk(v->mu);
      if (v->n_buffers == 0) spares.resize(kPrealloc);
      v->n_buffers += 1 + spares.size();
    }
    for (auto& b : spares)
      if (alloc_buffer(bytes, &b) != SAND_OK) b = PlanBuffer{};
    std::lock_guard<std::mutex> lk(v->mu);
    for (auto& b : spares)
      if (b.d) v->pool.push_back(b);
  } else {
    const uint64_t w0 = now_ns();
    cudaEventSynchronize(buf->done);    // kernels of the previous owner finished
    cudaEventSynchronize(buf->ready);   // its upload no longer reads the staging copy
    v->plan_buffer_wait_ns += now_ns() - w0;   // builder-side statistic (benign race)
  }
  auto* h = static_cast<uint8_t*>(buf->h);
  if (L.gb) std::memcpy(h, p.groups.data(), L.gb);
  if (L.ib) std::memcpy(h + L.off_i, p.items.data(), L.ib);
  if (L.db) std::memcpy(h + L.off_d, p.dests.data(), L.db);
  if (L.tb) std::memcpy(h + L.off_t, p.tasks.data(), L.tb);
  e = cudaMemcpyAsync(buf->d, buf->h, L.total, cudaMemcpyHostToDevice, v->upload_stream);
  if (e != cudaSuccess) return cuda_error(e, "cudaMemcpyAsync(plan)");
  e = cudaEventRecord(buf->ready, v->upload_stream);
  if (e != cudaSuccess) return cuda_error(e, "cudaEventRecord(plan ready)");
  auto* d = static_cast<uint8_t*>(buf->d);
  p.d_buf = buf->d;
  p.h_stage = buf->h;
  p.d_bytes = buf->bytes;
  p.last_use = buf->done;
  p.ready = buf->ready;
  p.ready_waited = nullptr;
  p.d_groups = reinterpret_cast<GroupParams*>(d);
  p.d_items = reinterpret_cast<WorkItem*>(d + L.off_i);
  p.d_dests = reinterpret_cast<uint32_t*>(d + L.off_d);
  p.d_tasks = reinterpret_cast<uint2*>(d + L.off_t);
  p.uploaded = true;
  return SAND_OK;
}

// Caller holds v->mu. Returns the cached plan, waiting for / building (and uploading) it as
// needed; *rc reports an upload failure (the plan is then returned without device copy).
std::shared_ptr<EpochPlan> get_plan(sand_view* v, std::unique_lock<std::mutex>& lk, uint64_t epoch, uint32_t rank,
                                    int* rc = nullptr) {
  const auto key = std::make_pair(epoch, rank);
  for (;;) {
    auto it = v->plans.find(key);
    if (it != v->plans.end()) {
      it->second->last_touch = ++v->touch;
      return it->second;
    }
    if (v->pending.count(key)) {
      if (rc) v->pending_waits++;
      v->cv.wait(lk);
      continue;
    }
    break;
  }
  v->pending[key] = true;
  std::shared_ptr<EpochPlan> plan;
  if (!v->spare_plans.empty()) {
    plan = std::move(v->spare_plans.back());
    v->spare_plans.pop_back();
  }
  lk.unlock();
  const uint64_t t0 = now_ns();
  plan = build_plan(*v, epoch, rank, std::move(plan));
  const uint64_t tb = now_ns();
  const PlanLayout L = plan_layout(*plan);
  lk.lock();
  v->plan_cpu_ns += tb - t0;
  PlanBuffer buf = take_buffer(v, L.total);
  lk.unlock();
  const int urc = upload_plan(v, *plan, &buf);
  const uint64_t t1 = now_ns();
  lk.lock();
  v->plan_build_ns += t1 - t0;
  v->pending.erase(key);
  if (rc) *rc = urc;
  if (urc != SAND_OK) {   // not cached: the next call rebuilds; the buffer returns to the pool
    if (buf.d) v->pool.push_back(buf);
    plan->uploaded = false;
    v->cv.notify_all();
    return plan;
  }
  v->plans_built++;
  plan->last_touch = ++v->touch;
  v->plans[key] = plan;
  while (v->plans.size() > kPlanCache) {   // evict the least recently used unpinned plan
    auto victim = v->plans.end();
    for (auto i = v->plans.begin(); i != v->plans.end(); ++i)
      if (i->first != key && i->second->pins == 0 &&
          (victim == v->plans.end() || i->second->last_touch < victim->second->last_touch))
        victim = i;
    if (victim == v->plans.end()) break;
    release_plan_device(v, *victim->second);
    if (victim->second.use_count() == 1) v->spare_plans.push_back(std::move(victim->second));
    v->plans.erase(victim);
  }
  v->cv.notify_all();
  return plan;
}

void worker_loop(sand_view* v) {
  std::unique_lock<std::mutex> lk(v->mu);
  for (;;) {
    v->cv.wait(lk, [v] { return v->stop || !v->queue.empty(); });
    if (v->stop) return;
    const auto key = v->queue.front();
    v->queue.pop_front();
    if (v->plans.count(key) || v->pending.count(key)) continue;
    get_plan(v, lk, key.first, key.second);
  }
}

size_t dtype_bytes(int32_t d) { return d == SAND_U8 ? 1 : (d == SAND_BF16 ? 2 : 4); }

}  // namespace
}  // namespace sand

extern "C" int sand_view_create(sand_store* s, const sand_view_spec* spec, sand_view** out) {
  if (!s || !spec || !out) return sand::set_error(SAND_EINVAL, "null argument");
  *out = nullptr;
  std::string why;
  int rc = sand::validate_spec(*spec, &why);
  if (rc != SAND_OK) return sand::set_error(rc, why);
  auto* v = new sand_view();
  v->store = s;
  v->info.spec = *spec;
  v->info.videos.assign(spec->videos, spec->videos + spec->n_videos);
  v->info.spec.videos = v->info.videos.data();
  {
    std::lock_guard<std::mutex> lk(s->mu);
    for (uint32_t id : v->info.videos) {
      auto it = s->videos.find(id);
      if (it == s->videos.end()) {
        delete v;
        return sand::set_error(SAND_ERANGE, "dataset video " + std::to_string(id) + " not in the store");
      }
      v->info.dims.push_back({id, it->second.n_frames, it->second.width, it->second.height});
      v->entries.push_back(&it->second);
    }
  }
  sand::derive_spec(&v->info);
  // per-video geometry checks: RRC boxes always fit; short side crops must fit the resized frame
  for (const auto& d : v->info.dims) {
    for (uint32_t k = 0; k < spec->n_views; ++k) {
      const sand_view_desc& vd = spec->views[k];
      if (vd.geom != SAND_GEOM_SHORTSIDE_CROP) continue;
      const uint64_t S = vd.short_side;
      const uint64_t Wp = d.width <= d.height ? S : d.width * S / d.height;
      const uint64_t Hp = d.width <= d.height ? d.height * S / d.width : S;
      if (Wp < vd.out_w || Hp < vd.out_h) {
        delete v;
        return sand::set_error(SAND_EINVAL, "short-side crop larger than the resized frame");
      }
    }
  }
  int max_h = 0, max_w = 0, max_r = 0;
  bool stencil = false;
  for (uint32_t k = 0; k < spec->n_views; ++k) {
    const sand_view_desc& vd = spec->views[k];
    sand::ViewConst& c = v->vconst[k];
    c.fold = 1;
    for (int ch = 0; ch < 3; ++ch) {   // normalisation constants in double, cast once (R#17)
      c.a[ch] = static_cast<float>(1.0 / (255.0 * vd.std[ch]));
      c.b[ch] = static_cast<float>(-vd.mean[ch] / vd.std[ch]);
      const double bf = static_cast<double>(c.b[ch]) - std::ldexp(static_cast<double>(c.a[ch]), 23);
      c.bf[ch] = static_cast<float>(bf);
      if (static_cast<double>(c.bf[ch]) != bf) c.fold = 0;
    }
    c.dtype = vd.out_dtype;
    c.T = static_cast<int32_t>(vd.clip_len);
    c.out_h = static_cast<int32_t>(vd.out_h);
    c.out_w = static_cast<int32_t>(vd.out_w);
    if (vd.rot_p > 0.0 || vd.blur_p > 0.0 || vd.jitter_p > 0.0) {
      stencil = true;
      max_h = std::max(max_h, static_cast<int>(vd.out_h));
      max_w = std::max(max_w, static_cast<int>(vd.out_w));
      if (vd.blur_p > 0.0) max_r = std::max(max_r, static_cast<int>((vd.blur_ksize - 1) / 2));
    }
  }
  cudaError_t e = cudaSetDevice(s->device);
  if (e != cudaSuccess) {
    delete v;
    return sand::cuda_error(e, "cudaSetDevice");
  }
  v->stencil_smem = stencil ? sand::stencil_smem_bytes(max_h, max_w, max_r) : 0;
  {   // k_plain CTA: frames of one clip group side by side, NQ threads per frame row
    uint32_t wmax = 4;
    for (uint32_t k = 0; k < spec->n_views; ++k) wmax = std::max(wmax, spec->views[k].out_w);
    const int cpt = sand::plain_cols_per_thread();
    v->pl_nq = static_cast<int>((wmax + cpt - 1) / cpt);
    v->pl_fpc = std::max(1, std::min(8, sand::plain_max_threads() / v->pl_nq));
  }
  rc = sand::configure_kernels(v->stencil_smem);
  if (rc != SAND_OK) {
    delete v;
    return rc;
  }
  e = cudaStreamCreateWithFlags(&v->upload_stream, cudaStreamNonBlocking);
  if (e != cudaSuccess) {
    delete v;
    return sand::cuda_error(e, "cudaStreamCreate(upload)");
  }
  s->live_views++;
  const int n_workers = 3;   // plan builders (epochs e + 1 .. e + kPlanAhead)
  for (int i = 0; i < n_workers; ++i) v->workers.emplace_back(sand::worker_loop, v);
  *out = v;
  return SAND_OK;
}

extern "C" int sand_view_output_desc(const sand_view* v, uint32_t k, sand_tensor_desc* out) {
  if (!v || !out) return sand::set_error(SAND_EINVAL, "null argument");
  if (k >= v->info.spec.n_views) return sand::set_error(SAND_ERANGE, "view index out of range");
  const sand_view_desc& d = v->info.spec.views[k];
  out->dims[0] = v->info.spec.batch_size;
  out->dims[1] = 3;
  out->dims[2] = d.clip_len;
  out->dims[3] = d.out_h;
  out->dims[4] = d.out_w;
  out->dtype = d.out_dtype;
  out->bytes = static_cast<uint64_t>(out->dims[0]) * 3 * d.clip_len * d.out_h * d.out_w * sand::dtype_bytes(d.out_dtype);
  return SAND_OK;
}

extern "C" int sand_view_iterations(const sand_view* v, uint64_t epoch, uint32_t rank, uint64_t* n) {
  (void)epoch;
  if (!v || !n) return sand::set_error(SAND_EINVAL, "null argument");
  const sand_view_spec& s = v->info.spec;
  if (rank >= s.world_size) return sand::set_error(SAND_EINVAL, "rank >= world_size");
  *n = sand::samples_per_rank(s.n_videos * s.samples_per_video, s.world_size, s.drop_last != 0) / s.batch_size;
  return SAND_OK;
}

extern "C" int sand_view_prefetch_epoch(sand_view* v, uint64_t epoch, uint32_t rank) {
  if (!v) return sand::set_error(SAND_EINVAL, "null argument");
  if (rank >= v->info.spec.world_size) return sand::set_error(SAND_EINVAL, "rank >= world_size");
  std::lock_guard<std::mutex> lk(v->mu);
  v->queue.push_back({epoch, rank});
  v->cv.notify_all();
  return SAND_OK;
}

static int read_batch_direct(sand_view* v, uint64_t epoch, uint32_t rank, const sand_batch_out* out);

namespace sand {
namespace {
// the pre-materialised slot holding (epoch, rank, iteration), or -1 (caller holds v->mu)
int find_slot(const sand_view* v, uint64_t epoch, uint32_t rank, uint64_t it) {
  for (size_t i = 0; i < v->pre.size(); ++i) {
    const auto& sl = v->pre[i];
    if (sl.busy && sl.epoch == epoch && sl.rank == rank && sl.iteration == it) return static_cast<int>(i);
  }
  return -1;
}
void free_slots(sand_view* v) {
  for (auto& sl : v->pre) {
    if (sl.done) {
      cudaEventSynchronize(sl.done);
      cudaEventDestroy(sl.done);
    }
    if (sl.consumed) {
      cudaEventSynchronize(sl.consumed);
      cudaEventDestroy(sl.consumed);
    }
    cudaFree(sl.buf);
  }
  v->pre.clear();
}
}  // namespace
}  // namespace sand

extern "C" int sand_view_set_prematerialize(sand_view* v, uint32_t slots) {
  if (!v) return sand::set_error(SAND_EINVAL, "null argument");
  std::lock_guard<std::mutex> lk(v->mu);
  cudaError_t e = cudaSetDevice(v->store->device);
  if (e != cudaSuccess) return sand::cuda_error(e, "cudaSetDevice");
  sand::free_slots(v);
  if (slots == 0) return SAND_OK;
  if (!v->pre_stream) {
    int lo = 0, hi = 0;
    cudaDeviceGetStreamPriorityRange(&lo, &hi);   // lo = least priority
    e = cudaStreamCreateWithPriority(&v->pre_stream, cudaStreamNonBlocking, lo);
    if (e != cudaSuccess) return sand::cuda_error(e, "cudaStreamCreateWithPriority(prematerialize)");
  }
  size_t total = 0;
  for (uint32_t k = 0; k < v->info.spec.n_views; ++k) {
    sand_tensor_desc td;
    sand_view_output_desc(v, k, &td);
    v->pre_view_off[k] = total;
    v->pre_view_bytes[k] = td.bytes;
    total += (td.bytes + 255) / 256 * 256;
  }
  v->pre.resize(slots);
  for (auto& sl : v->pre) {
    e = cudaMalloc(&sl.buf, total);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&sl.done, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&sl.consumed, cudaEventDisableTiming);
    if (e != cudaSuccess) {
      sand::free_slots(v);
      return sand::cuda_error(e, "pre-materialisation buffers");
    }
  }
  return SAND_OK;
}

extern "C" int sand_view_prematerialize(sand_view* v, uint64_t epoch, uint32_t rank, uint64_t iteration) {
  if (!v) return sand::set_error(SAND_EINVAL, "null argument");
  sand_batch_out out{};
  int slot = -1;
  {
    std::lock_guard<std::mutex> lk(v->mu);
    if (v->pre.empty()) return sand::set_error(SAND_EINVAL, "pre-materialisation not configured");
    if (sand::find_slot(v, epoch, rank, iteration) >= 0) return SAND_OK;   // already under way
    for (size_t i = 0; i < v->pre.size(); ++i)
      if (!v->pre[i].busy) {
        slot = static_cast<int>(i);
        break;
      }
    if (slot < 0) return sand::set_error(SAND_EBUSY, "every pre-materialisation slot holds an unread batch");
    auto& sl = v->pre[slot];
    // the slot's previous batch may still be being copied out / used by its reader
    if (sl.consumed_pending) {
      cudaError_t e = cudaStreamWaitEvent(v->pre_stream, sl.consumed, 0);
      if (e != cudaSuccess) return sand::cuda_error(e, "cudaStreamWaitEvent(slot consumed)");
      sl.consumed_pending = false;
    }
    out.iteration = iteration;
    out.stream = v->pre_stream;
    for (uint32_t k = 0; k < v->info.spec.n_views; ++k) out.data[k] = sl.buf + v->pre_view_off[k];
    sl.busy = true;   // reserved while the kernels are enqueued
    sl.epoch = epoch;
    sl.rank = rank;
    sl.iteration = iteration;
  }
  const int rc = read_batch_direct(v, epoch, rank, &out);
  std::lock_guard<std::mutex> lk(v->mu);
  auto& sl = v->pre[slot];
  if (rc != SAND_OK) {
    sl.busy = false;
    return rc;
  }
  cudaError_t e = cudaEventRecord(sl.done, v->pre_stream);
  if (e != cudaSuccess) {
    sl.busy = false;
    return sand::cuda_error(e, "cudaEventRecord(prematerialized)");
  }
  v->pre_made++;
  return SAND_OK;
}

extern "C" int sand_view_acquire_batch(sand_view* v, uint64_t epoch, uint32_t rank, uint64_t iteration,
                                       sand_stream_t stream, void* data_out[SAND_MAX_VIEWS]) {
  if (!v || !data_out) return sand::set_error(SAND_EINVAL, "null argument");
  std::lock_guard<std::mutex> lk(v->mu);
  const int i = sand::find_slot(v, epoch, rank, iteration);
  if (i < 0 || v->pre[i].acquired) return sand::set_error(SAND_ERANGE, "batch is not pre-materialised");
  auto& sl = v->pre[i];
  cudaError_t e = cudaStreamWaitEvent(static_cast<cudaStream_t>(stream), sl.done, 0);
  if (e != cudaSuccess) return sand::cuda_error(e, "cudaStreamWaitEvent(prematerialized)");
  for (uint32_t k = 0; k < SAND_MAX_VIEWS; ++k)
    data_out[k] = k < v->info.spec.n_views ? static_cast<void*>(sl.buf + v->pre_view_off[k]) : nullptr;
  sl.acquired = true;
  v->pre_served++;
  return SAND_OK;
}

extern "C" int sand_view_release_batch(sand_view* v, uint64_t epoch, uint32_t rank, uint64_t iteration,
                                       sand_stream_t stream) {
  if (!v) return sand::set_error(SAND_EINVAL, "null argument");
  std::lock_guard<std::mutex> lk(v->mu);
  const int i = sand::find_slot(v, epoch, rank, iteration);
  if (i < 0 || !v->pre[i].acquired) return sand::set_error(SAND_ERANGE, "batch was not acquired");
  auto& sl = v->pre[i];
  cudaError_t e = cudaEventRecord(sl.consumed, static_cast<cudaStream_t>(stream));
  if (e != cudaSuccess) return sand::cuda_error(e, "cudaEventRecord(slot consumed)");
  sl.consumed_pending = true;
  sl.acquired = false;
  sl.busy = false;
  return SAND_OK;
}

extern "C" int sand_view_read_batch(sand_view* v, uint64_t epoch, uint32_t rank, const sand_batch_out* out) {
  if (!v || !out) return sand::set_error(SAND_EINVAL, "null argument");
  {   // a pre-materialised batch: wait for it and copy it out (stream-ordered)
    std::lock_guard<std::mutex> lk(v->mu);
    const int i = v->pre.empty() ? -1 : sand::find_slot(v, epoch, rank, out->iteration);
    if (i >= 0 && !v->pre[i].acquired) {
      auto& sl = v->pre[i];
      auto stream = static_cast<cudaStream_t>(out->stream);
      cudaError_t e = cudaStreamWaitEvent(stream, sl.done, 0);
      for (uint32_t k = 0; k < v->info.spec.n_views && e == cudaSuccess; ++k) {
        if (!out->data[k]) return sand::set_error(SAND_EINVAL, "null output pointer");
        e = cudaMemcpyAsync(out->data[k], sl.buf + v->pre_view_off[k], v->pre_view_bytes[k], cudaMemcpyDeviceToDevice,
                            stream);
      }
      if (e == cudaSuccess) e = cudaEventRecord(sl.consumed, stream);
      if (e != cudaSuccess) return sand::cuda_error(e, "serving a pre-materialised batch");
      sl.consumed_pending = true;
      sl.busy = false;
      v->pre_served++;
      return SAND_OK;
    }
  }
  return read_batch_direct(v, epoch, rank, out);
}

static int read_batch_direct(sand_view* v, uint64_t epoch, uint32_t rank, const sand_batch_out* out) {
  if (!v || !out) return sand::set_error(SAND_EINVAL, "null argument");
  const sand_view_spec& s = v->info.spec;
  if (rank >= s.world_size) return sand::set_error(SAND_EINVAL, "rank >= world_size");
  for (uint32_t k = 0; k < s.n_views; ++k) {
    if (!out->data[k]) return sand::set_error(SAND_EINVAL, "null output pointer");
    if (reinterpret_cast<uintptr_t>(out->data[k]) % 16 != 0) return sand::set_error(SAND_EINVAL, "output not 16 B aligned");
  }
  auto stream = static_cast<cudaStream_t>(out->stream);
  const uint64_t t0 = sand::now_ns();
  std::unique_lock<std::mutex> lk(v->mu);
  v->lock_wait_ns += sand::now_ns() - t0;
  int urc = SAND_OK;
  auto plan = sand::get_plan(v, lk, epoch, rank, &urc);
  const uint64_t t1 = sand::now_ns();
  v->plan_wait_ns += t1 - t0;
  if (out->iteration >= plan->iterations) return sand::set_error(SAND_ERANGE, "iteration out of range");
  cudaError_t e = cudaSetDevice(v->store->device);
  if (e != cudaSuccess) return sand::cuda_error(e, "cudaSetDevice");
  if (!plan->uploaded) return urc != SAND_OK ? urc : sand::set_error(SAND_ECUDA, "plan has no device copy");
  if (plan->ready_waited != stream) {   // order the caller's stream after the plan upload
    e = cudaStreamWaitEvent(stream, plan->ready, 0);
    if (e != cudaSuccess) return sand::cuda_error(e, "cudaStreamWaitEvent(plan ready)");
    plan->ready_waited = stream;
  }
  const uint64_t it = out->iteration;
  const uint32_t ib = plan->item_begin[it], ie = plan->item_begin[it + 1];
  // plan the next epochs on the builder threads while this one is consumed
  // (pre-materialisation of the plan, the analogue of the paper's pre-materialisation
  // threads)
  if (it == 0) {
    for (uint64_t ahead = 1; ahead <= sand::kPlanAhead; ++ahead) {
      const auto next = std::make_pair(epoch + ahead, rank);
      if (!v->plans.count(next) && !v->pending.count(next) &&
          std::find(v->queue.begin(), v->queue.end(), next) == v->queue.end()) {
        v->queue.push_back(next);
        v->cv.notify_one();
      }
    }
  }
  sand_store* st = v->store;
  {
    std::lock_guard<std::mutex> slk(st->mu);
    for (uint32_t i = plan->fetch_begin[it]; i < plan->fetch_begin[it + 1]; ++i) {
      if (!plan->fetch_entry[i]->present[plan->fetch_keys[i].second]) {
        const auto& key = plan->fetch_keys[i];
        return sand::set_error(SAND_ENOENT, "frame " + std::to_string(key.second) + " of video " +
                                                std::to_string(key.first) + " is not in the store");
      }
    }
    // frames put since this stream last waited: order the kernel after their copies
    if (st->put_seq > 0 && (st->put_seq != v->put_seq_seen || stream != v->put_stream_seen)) {
      e = cudaStreamWaitEvent(stream, st->last_put, 0);
      if (e != cudaSuccess) return sand::cuda_error(e, "cudaStreamWaitEvent(last_put)");
      v->put_seq_seen = st->put_seq;
      v->put_stream_seen = stream;
    }
  }
  // bound the read-ahead: at most kInflight batches of this view are queued on the GPU. An
  // unbounded run-ahead keeps many epoch plans alive at once (more plan buffers, allocations
  // and driver locks while batches are being read) for no gain.
  const size_t slot = static_cast<size_t>(v->batches % sand::kInflight);
  if (v->inflight.empty()) {
    v->inflight.resize(sand::kInflight, nullptr);
    for (auto& ev : v->inflight) {
      e = cudaEventCreateWithFlags(&ev, cudaEventDisableTiming);
      if (e != cudaSuccess) return sand::cuda_error(e, "cudaEventCreate(inflight)");
    }
  }
  if (v->batches >= sand::kInflight) {
    // the plan is pinned while the lock is dropped: a builder thread cannot evict it and
    // recycle its device buffer before the kernel below has been launched
    plan->pins++;
    lk.unlock();
    e = cudaEventSynchronize(v->inflight[slot]);
    lk.lock();
    plan->pins--;
    if (e != cudaSuccess) return sand::cuda_error(e, "cudaEventSynchronize(inflight)");
    if (!plan->uploaded) return sand::set_error(SAND_ECUDA, "plan lost its device copy");
  }
  sand::LaunchParams lp{};
  lp.slab = st->slab;
  lp.items = plan->d_items + ib;
  lp.n_items = ie - ib;
  lp.groups = plan->d_groups;
  lp.dests = plan->d_dests;
  lp.n_views = s.n_views;
  lp.batch = s.batch_size;
  lp.tasks = plan->d_tasks;
  lp.cm = sand::color_matrix(s.views[0].color_matrix);
  for (uint32_t k = 0; k < s.n_views; ++k) {
    lp.out[k] = out->data[k];
    lp.views[k] = v->vconst[k];
  }
  int launched = 0;
  const sand::BatchShape& bshape = plan->shapes[it];
  const int classes = (bshape.n_mild > 0) + (bshape.n_direct > bshape.n_mild) + (lp.n_items > bshape.n_direct);
  if (classes > 1 && !v->aux_stream) {
    e = cudaStreamCreateWithFlags(&v->aux_stream, cudaStreamNonBlocking);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&v->fork_ev, cudaEventDisableTiming);
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&v->join_ev, cudaEventDisableTiming);
    if (e != cudaSuccess) return sand::cuda_error(e, "aux stream for the direct kernel");
  }
  sand::ClassEvents cev{};
  if (v->timing) {   // measurement only: an event pair per class from the view's pool
    for (int c = 0; c < 3; ++c)
      for (cudaEvent_t* ev : {&cev.start[c], &cev.end[c]}) {
        if (v->free_events.empty()) {
          e = cudaEventCreate(ev);
          if (e != cudaSuccess) return sand::cuda_error(e, "cudaEventCreate(timing)");
        } else {
          *ev = v->free_events.back();
          v->free_events.pop_back();
        }
      }
  }
  bool cached = false;
  int rc = sand::objcache_read(v, *plan, it, lp, stream, &launched, &cached);   // f2 object cache, if configured
  if (rc == SAND_OK && !cached)
    rc = sand::launch_materialize(lp, bshape, v->stencil_smem, v->pl_fpc, v->pl_nq, stream, v->aux_stream, v->fork_ev,
                                  v->join_ev, &launched, v->timing ? &cev : nullptr);
  if (v->timing)
    for (int c = 0; c < 3; ++c) {
      if (cev.used[c] && rc == SAND_OK) {
        v->timed.push_back({c, cev.start[c], cev.end[c]});
      } else {
        v->free_events.push_back(cev.start[c]);
        v->free_events.push_back(cev.end[c]);
      }
    }
  if (rc != SAND_OK) return rc;
  e = cudaEventRecord(plan->last_use, stream);
  if (e == cudaSuccess) e = cudaEventRecord(v->inflight[slot], stream);
  if (e != cudaSuccess) return sand::cuda_error(e, "cudaEventRecord");
  {
    std::lock_guard<std::mutex> slk(st->mu);
    for (uint32_t i = plan->fetch_begin[it]; i < plan->fetch_begin[it + 1]; ++i) {
      sand::VideoEntry* ve = plan->fetch_entry[i];
      ve->fetches[plan->fetch_keys[i].second] += 1;
      ve->uses[plan->fetch_keys[i].second] += plan->fetch_uses[i];
    }
    st->batches++;
  }
  v->batches++;
  v->launches += static_cast<uint64_t>(launched);
  v->work_items += lp.n_items;
  v->read_ns += sand::now_ns() - t0;
  return SAND_OK;
}

extern "C" int sand_view_get_meta(sand_view* v, uint64_t epoch, uint32_t rank, uint64_t iteration,
                                  sand_clip_meta* out) {
  if (!v || !out) return sand::set_error(SAND_EINVAL, "null argument");
  if (rank >= v->info.spec.world_size) return sand::set_error(SAND_EINVAL, "rank >= world_size");
  std::unique_lock<std::mutex> lk(v->mu);
  auto plan = sand::get_plan(v, lk, epoch, rank);
  if (iteration >= plan->iterations) return sand::set_error(SAND_ERANGE, "iteration out of range");
  const uint32_t B = v->info.spec.batch_size;
  std::memcpy(out, plan->metas.data() + iteration * B, sizeof(sand_clip_meta) * B);
  return SAND_OK;
}

// Algorithmic source bytes of a batch: distinct 32 B sectors of the
// source rows touched by any bilinear tap, deduplicated across views, groups and
// clips that share a (video, frame); rows assumed 32 B aligned (the store's pitch
// is a multiple of 64 B). Taps follow the same fp32 coordinate rule as the kernel.
// cls < 0: every item; else only the items of that class (SAND_N_CLASSES).
static int batch_bytes_impl(sand_view* v, uint64_t epoch, uint32_t rank, uint64_t iteration, int cls,
                            sand_batch_bytes* out) {
  if (!v || !out) return sand::set_error(SAND_EINVAL, "null argument");
  if (rank >= v->info.spec.world_size) return sand::set_error(SAND_EINVAL, "rank >= world_size");
  if (cls >= SAND_N_CLASSES) return sand::set_error(SAND_EINVAL, "class out of range");
  std::unique_lock<std::mutex> lk(v->mu);
  auto plan = sand::get_plan(v, lk, epoch, rank);
  lk.unlock();
  if (iteration >= plan->iterations) return sand::set_error(SAND_ERANGE, "iteration out of range");
  const sand_view_spec& s = v->info.spec;
  std::memset(out, 0, sizeof(*out));
  const uint32_t ib = plan->item_begin[iteration], ie = plan->item_begin[iteration + 1];
  const sand::BatchShape& shape = plan->shapes[iteration];
  auto class_of = [&](uint32_t i) {
    const uint32_t r = i - ib;
    return r < shape.n_mild ? 0 : (r < shape.n_direct ? 1 : 2);
  };
  // group the selected items by source frame; output bytes and uses from their destinations
  std::map<uint64_t, std::vector<uint32_t>> by_frame;
  for (uint32_t i = ib; i < ie; ++i) {
    if (cls >= 0 && class_of(i) != cls) continue;
    const sand::WorkItem& w = plan->items[i];
    by_frame[w.y_off].push_back(i);
    for (uint32_t d = 0; d < w.n_dest; ++d) {
      const sand_view_desc& vd = s.views[plan->dests[w.dest_begin + d] >> 24];
      out->out_bytes += 3ull * vd.out_h * vd.out_w * sand::dtype_bytes(vd.out_dtype);
    }
    out->uses += w.n_dest;
  }
  for (auto& kv : by_frame) {
    const sand::WorkItem& w0 = plan->items[kv.second[0]];
    const uint32_t W = w0.src_w, H = w0.src_h, nsec = (W + 31) / 32;
    std::vector<uint8_t> ysec(static_cast<size_t>(H) * nsec, 0), uvsec(static_cast<size_t>(H / 2) * nsec, 0);
    for (uint32_t i : kv.second) {
      const sand::GroupParams& g = plan->groups[plan->items[i].gp];
      auto taps = [](float sc, int off, int n_out, int lim, int org, std::vector<uint8_t>& mark) {
        for (int o = 0; o < n_out; ++o) {
          int i0, i1;
          float l;
          sand::tap_ref(sc, off, o, lim, org, &i0, &i1, &l);
          mark[i0] = 1;
          mark[i1] = 1;
        }
      };
      std::vector<uint8_t> cols(W, 0), rows(H, 0);
      taps(g.sc_x, g.off_x, g.out_w, g.lim_x, g.org_x, cols);
      taps(g.sc_y, g.off_y, g.out_h, g.lim_y, g.org_y, rows);
      std::vector<uint8_t> ymask(nsec, 0), uvmask(nsec, 0);
      for (uint32_t x = 0; x < W; ++x)
        if (cols[x]) {
          ymask[x / 32] = 1;
          uvmask[(x & ~1u) / 32] = 1;
          uvmask[((x & ~1u) + 1) / 32] = 1;
        }
      for (uint32_t y = 0; y < H; ++y)
        if (rows[y])
          for (uint32_t c = 0; c < nsec; ++c) {
            ysec[static_cast<size_t>(y) * nsec + c] |= ymask[c];
            uvsec[static_cast<size_t>(y / 2) * nsec + c] |= uvmask[c];
          }
    }
    for (uint8_t b : ysec) out->src_sectors += b;
    for (uint8_t b : uvsec) out->src_sectors += b;
  }
  out->src_bytes = out->src_sectors * 32;
  if (cls < 0) {
    for (uint32_t i = plan->fetch_begin[iteration]; i < plan->fetch_begin[iteration + 1]; ++i) out->fetches += 1;
  } else {
    std::map<uint64_t, int> frames;
    for (const auto& kv : by_frame) frames[kv.first] = 1;
    out->fetches = frames.size();
  }
  return SAND_OK;
}

extern "C" int sand_view_batch_bytes(sand_view* v, uint64_t epoch, uint32_t rank, uint64_t iteration,
                                     sand_batch_bytes* out) {
  return batch_bytes_impl(v, epoch, rank, iteration, -1, out);
}

extern "C" int sand_view_batch_bytes_class(sand_view* v, uint64_t epoch, uint32_t rank, uint64_t iteration, uint32_t cls,
                                           sand_batch_bytes* out) {
  if (cls >= SAND_N_CLASSES) return sand::set_error(SAND_EINVAL, "class out of range");
  return batch_bytes_impl(v, epoch, rank, iteration, static_cast<int>(cls), out);
}

extern "C" int sand_view_set_timing(sand_view* v, int on) {
  if (!v) return sand::set_error(SAND_EINVAL, "null argument");
  std::lock_guard<std::mutex> lk(v->mu);
  v->timing = on != 0;
  return SAND_OK;
}

extern "C" int sand_view_class_times(sand_view* v, double ms[SAND_N_CLASSES], uint64_t launches[SAND_N_CLASSES]) {
  if (!v || !ms || !launches) return sand::set_error(SAND_EINVAL, "null argument");
  std::lock_guard<std::mutex> lk(v->mu);
  cudaError_t e = cudaSetDevice(v->store->device);
  if (e != cudaSuccess) return sand::cuda_error(e, "cudaSetDevice");
  for (const auto& t : v->timed) {
    e = cudaEventSynchronize(t.end);
    float x = 0.f;
    if (e == cudaSuccess) e = cudaEventElapsedTime(&x, t.start, t.end);
    if (e != cudaSuccess) return sand::cuda_error(e, "class timing events");
    v->class_ms[t.cls] += x;
    v->class_launches[t.cls] += 1;
    v->free_events.push_back(t.start);
    v->free_events.push_back(t.end);
  }
  v->timed.clear();
  for (int c = 0; c < SAND_N_CLASSES; ++c) {
    ms[c] = v->class_ms[c];
    launches[c] = v->class_launches[c];
    v->class_ms[c] = 0;
    v->class_launches[c] = 0;
  }
  return SAND_OK;
}

extern "C" int sand_view_get_stats(const sand_view* v, sand_view_stats* out) {
  if (!v || !out) return sand::set_error(SAND_EINVAL, "null argument");
  out->batches = v->batches;
  out->kernel_launches = v->launches;
  out->plans_built = v->plans_built;
  out->work_items = v->work_items;
  out->plan_build_ns = v->plan_build_ns;
  out->plan_wait_ns = v->plan_wait_ns;
  out->read_ns = v->read_ns;
  out->plan_cpu_ns = v->plan_cpu_ns;
  out->plan_buffer_wait_ns = v->plan_buffer_wait_ns;
  out->lock_wait_ns = v->lock_wait_ns;
  out->pending_waits = v->pending_waits;
  return SAND_OK;
}

extern "C" int sand_view_destroy(sand_view* v) {
  if (!v) return SAND_OK;
  {
    std::lock_guard<std::mutex> lk(v->mu);
    v->stop = true;
    v->cv.notify_all();
  }
  for (auto& w : v->workers)
    if (w.joinable()) w.join();
  cudaSetDevice(v->store->device);
  for (auto& kv : v->plans) sand::release_plan_device(v, *kv.second);
  sand::free_pool(v);
  if (v->upload_stream) cudaStreamDestroy(v->upload_stream);
  if (v->aux_stream) cudaStreamDestroy(v->aux_stream);
  if (v->fork_ev) cudaEventDestroy(v->fork_ev);
  if (v->join_ev) cudaEventDestroy(v->join_ev);
  for (auto& ev : v->inflight)
    if (ev) cudaEventDestroy(ev);
  for (auto& t : v->timed) {
    cudaEventDestroy(t.start);
    cudaEventDestroy(t.end);
  }
  for (auto& ev : v->free_events) cudaEventDestroy(ev);
  sand::free_slots(v);
  if (v->pre_stream) cudaStreamDestroy(v->pre_stream);
  sand::objcache_free(v);
  v->store->live_views--;
  delete v;
  return SAND_OK;
}
