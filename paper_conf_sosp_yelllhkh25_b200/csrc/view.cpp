// view.cpp — the view group: spec validation, epoch plans, read / getxattr / close
// (SAND view abstraction §5.1; POSIX API Table 2).
//
// Plans are built per (epoch, rank) on the host — synchronously on first use or
// ahead of time on a worker thread (sand_view_prefetch_epoch; the plan analogue of
// the paper's pre-materialisation threads) — and uploaded once, so a read
// is a presence check plus one kernel launch on the caller's stream.
#include <cuda_runtime.h>

#include <algorithm>
#include <cmath>
#include <cstring>

#include "internal.h"

namespace sand {
namespace {

constexpr size_t kPlanCache = 4;
constexpr double kPi = 3.14159265358979323846;

struct FrameBase {
  uint64_t offset, frame_stride;
  uint32_t pitch;
};

FrameBase frame_base(const sand_store* s, uint32_t video) {
  const VideoEntry& v = s->videos.at(video);
  return {v.offset, v.frame_stride, v.pitch};
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
  return g;
}

}  // namespace

std::shared_ptr<EpochPlan> build_plan(const sand_view& v, uint64_t epoch, uint32_t rank) {
  const SpecInfo& info = v.info;
  const sand_view_spec& s = info.spec;
  const uint32_t B = s.batch_size;
  const uint32_t nG = static_cast<uint32_t>(info.groups.size());
  auto plan = std::make_shared<EpochPlan>();
  plan->epoch = epoch;
  plan->rank = rank;
  const std::vector<uint32_t> clips = rank_clips(info, epoch, rank);
  plan->iterations = clips.size() / B;
  const uint64_t n_clips = plan->iterations * B;
  plan->metas.resize(n_clips);
  plan->groups.resize(n_clips * nG);
  plan->item_begin.push_back(0);
  plan->fetch_begin.push_back(0);
  int32_t common_dtype = s.views[0].out_dtype;
  int32_t even_wo = 1;
  for (uint32_t k = 0; k < s.n_views; ++k) {
    if (s.views[k].out_dtype != common_dtype) common_dtype = -1;
    if (s.views[k].out_w & 1u) even_wo = 0;
  }
  for (uint64_t it = 0; it < plan->iterations; ++it) {
    BatchShape shape{};
    shape.dtype = common_dtype;
    shape.even_wo = even_wo;
    std::vector<std::pair<uint64_t, uint32_t>> fetch;   // ((video<<32)|frame, uses)
    for (uint32_t b = 0; b < B; ++b) {
      const uint64_t slot = it * B + b;
      sand_clip_meta& m = plan->metas[slot];
      const uint32_t clip = clips[slot];
      plan_clip(info, epoch, clip, &m);
      const VideoDims& dim = info.dims[clip / s.samples_per_video];
      const FrameBase fb = frame_base(v.store, dim.id);
      for (uint32_t gi = 0; gi < nG; ++gi) {
        const uint32_t q = info.groups[gi];
        plan->groups[slot * nG + gi] = group_params(s.views[info.leader[q]], m, q, dim.width, dim.height);
      }
      // unique source frames of the clip, in order of first use
      std::vector<uint32_t> uniq;
      for (uint32_t k = 0; k < s.n_views; ++k)
        for (uint32_t t = 0; t < s.views[k].clip_len; ++t)
          if (std::find(uniq.begin(), uniq.end(), m.frames[k][t]) == uniq.end()) uniq.push_back(m.frames[k][t]);
      for (uint32_t f : uniq) {
        uint32_t uses = 0;
        for (uint32_t gi = 0; gi < nG; ++gi) {
          const uint32_t q = info.groups[gi];
          WorkItem w{};
          w.dest_begin = static_cast<uint32_t>(plan->dests.size());
          for (uint32_t k = 0; k < s.n_views; ++k) {
            if (s.views[k].spatial_group != q) continue;
            for (uint32_t t = 0; t < s.views[k].clip_len; ++t)
              if (m.frames[k][t] == f) plan->dests.push_back(pack_dest(k, t, b));
          }
          w.n_dest = static_cast<uint32_t>(plan->dests.size()) - w.dest_begin;
          if (w.n_dest == 0) continue;
          uses += w.n_dest;
          w.y_off = fb.offset + fb.frame_stride * f;
          w.pitch = fb.pitch;
          w.src_w = dim.width;
          w.src_h = dim.height;
          w.gp = static_cast<uint32_t>(slot * nG + gi);
          w.clip_slot = b;
          w.group = q;
          const GroupParams& g = plan->groups[w.gp];
          w.flags = (g.rot_on || g.blur_on) ? 1u : 0u;
          if (w.flags) {
            shape.has_stencil = 1;
            shape.st_max_wo = std::max(shape.st_max_wo, g.out_w);
            shape.st_max_ho = std::max(shape.st_max_ho, g.out_h);
            const int cols = std::min(2 * g.out_w, static_cast<int>(std::ceil(static_cast<double>(g.sc_x) * g.out_w)) + 3);
            shape.st_cols_bound = std::max(shape.st_cols_bound, cols);
            shape.st_max_scy = std::max(shape.st_max_scy, g.sc_y);
          } else {
            shape.has_direct = 1;
            shape.max_wo = std::max(shape.max_wo, g.out_w);
            shape.max_ho = std::max(shape.max_ho, g.out_h);
            const int cols = std::min(2 * g.out_w, static_cast<int>(std::ceil(static_cast<double>(g.sc_x) * g.out_w)) + 3);
            shape.cols_bound = std::max(shape.cols_bound, cols);
            shape.max_scy = std::max(shape.max_scy, g.sc_y);
          }
          plan->items.push_back(w);
        }
        fetch.push_back({(static_cast<uint64_t>(dim.id) << 32) | f, uses});
      }
    }
    // batch-unique (video, frame): merge clips that share a source frame
    std::sort(fetch.begin(), fetch.end());
    for (size_t i = 0; i < fetch.size();) {
      size_t j = i;
      uint32_t uses = 0;
      while (j < fetch.size() && fetch[j].first == fetch[i].first) uses += fetch[j++].second;
      plan->fetch_keys.push_back({static_cast<uint32_t>(fetch[i].first >> 32), static_cast<uint32_t>(fetch[i].first)});
      plan->fetch_uses.push_back(uses);
      i = j;
    }
    plan->fetch_begin.push_back(static_cast<uint32_t>(plan->fetch_keys.size()));
    plan->item_begin.push_back(static_cast<uint32_t>(plan->items.size()));
    plan->shapes.push_back(shape);
  }
  return plan;
}

namespace {

// return a plan's buffers to the view's pool (its kernels finish before the pool hands the
// buffer out again: the pool waits on the buffer's event, which is long done by then)
void release_plan_device(sand_view* v, EpochPlan& p) {
  if (p.d_buf) {
    PlanBuffer b;
    b.d = p.d_buf;
    b.h = p.h_stage;
    b.bytes = p.d_bytes;
    b.done = p.last_use;
    v->pool.push_back(b);
  } else if (p.last_use) {
    cudaEventDestroy(p.last_use);
  }
  p.d_buf = p.h_stage = nullptr;
  p.last_use = nullptr;
  p.uploaded = false;
}

void free_pool(sand_view* v) {
  for (auto& b : v->pool) {
    if (b.done) {
      cudaEventSynchronize(b.done);
      cudaEventDestroy(b.done);
    }
    cudaFree(b.d);
    cudaFreeHost(b.h);
  }
  v->pool.clear();
}

int upload_plan(sand_view* v, EpochPlan& p, cudaStream_t stream) {
  const size_t gb = p.groups.size() * sizeof(GroupParams);
  const size_t ib = p.items.size() * sizeof(WorkItem);
  const size_t db = p.dests.size() * sizeof(uint32_t);
  const size_t off_i = (gb + 255) / 256 * 256;
  const size_t off_d = off_i + (ib + 255) / 256 * 256;
  const size_t total = std::max<size_t>(off_d + db, 256);
  // smallest pooled buffer that fits, else a new one with headroom
  int best = -1;
  for (size_t i = 0; i < v->pool.size(); ++i)
    if (v->pool[i].bytes >= total && (best < 0 || v->pool[i].bytes < v->pool[best].bytes)) best = (int)i;
  PlanBuffer buf;
  if (best >= 0) {
    buf = v->pool[best];
    v->pool.erase(v->pool.begin() + best);
    if (buf.done) cudaEventSynchronize(buf.done);   // the previous owner's kernels are done
  } else {
    buf.bytes = total + total / 4;
    cudaError_t e = cudaMalloc(&buf.d, buf.bytes);
    if (e != cudaSuccess) return cuda_error(e, "cudaMalloc(plan)");
    e = cudaMallocHost(&buf.h, buf.bytes);
    if (e != cudaSuccess) {
      cudaFree(buf.d);
      return cuda_error(e, "cudaMallocHost(plan)");
    }
    e = cudaEventCreateWithFlags(&buf.done, cudaEventDisableTiming);
    if (e != cudaSuccess) return cuda_error(e, "cudaEventCreate");
  }
  auto* h = static_cast<uint8_t*>(buf.h);
  if (gb) std::memcpy(h, p.groups.data(), gb);
  if (ib) std::memcpy(h + off_i, p.items.data(), ib);
  if (db) std::memcpy(h + off_d, p.dests.data(), db);
  cudaError_t e = cudaMemcpyAsync(buf.d, buf.h, total, cudaMemcpyHostToDevice, stream);
  if (e != cudaSuccess) return cuda_error(e, "cudaMemcpyAsync(plan)");
  auto* d = static_cast<uint8_t*>(buf.d);
  p.d_buf = buf.d;
  p.h_stage = buf.h;
  p.d_bytes = buf.bytes;
  p.last_use = buf.done;
  p.d_groups = reinterpret_cast<GroupParams*>(d);
  p.d_items = reinterpret_cast<WorkItem*>(d + off_i);
  p.d_dests = reinterpret_cast<uint32_t*>(d + off_d);
  p.uploaded = true;
  return SAND_OK;
}

// Caller holds v->mu. Returns the cached plan, waiting for / building it as needed.
std::shared_ptr<EpochPlan> get_plan(sand_view* v, std::unique_lock<std::mutex>& lk, uint64_t epoch, uint32_t rank) {
  const auto key = std::make_pair(epoch, rank);
  for (;;) {
    auto it = v->plans.find(key);
    if (it != v->plans.end()) {
      it->second->last_touch = ++v->touch;
      return it->second;
    }
    if (v->pending.count(key)) {
      v->cv.wait(lk);
      continue;
    }
    break;
  }
  v->pending[key] = true;
  lk.unlock();
  auto plan = build_plan(*v, epoch, rank);
  lk.lock();
  v->pending.erase(key);
  v->plans_built++;
  plan->last_touch = ++v->touch;
  v->plans[key] = plan;
  while (v->plans.size() > kPlanCache) {   // evict the least recently used plan
    auto victim = v->plans.begin();
    for (auto i = v->plans.begin(); i != v->plans.end(); ++i)
      if (i->second->last_touch < victim->second->last_touch) victim = i;
    if (victim->first == key) break;
    release_plan_device(v, *victim->second);
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
    for (int ch = 0; ch < 3; ++ch) {   // normalisation constants in double, cast once (R#17)
      c.a[ch] = static_cast<float>(1.0 / (255.0 * vd.std[ch]));
      c.b[ch] = static_cast<float>(-vd.mean[ch] / vd.std[ch]);
    }
    c.dtype = vd.out_dtype;
    c.T = static_cast<int32_t>(vd.clip_len);
    c.out_h = static_cast<int32_t>(vd.out_h);
    c.out_w = static_cast<int32_t>(vd.out_w);
    if (vd.rot_p > 0.0 || vd.blur_p > 0.0) {
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
  rc = sand::configure_kernels(v->stencil_smem);
  if (rc != SAND_OK) {
    delete v;
    return rc;
  }
  s->live_views++;
  v->worker = std::thread(sand::worker_loop, v);
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

extern "C" int sand_view_read_batch(sand_view* v, uint64_t epoch, uint32_t rank, const sand_batch_out* out) {
  if (!v || !out) return sand::set_error(SAND_EINVAL, "null argument");
  const sand_view_spec& s = v->info.spec;
  if (rank >= s.world_size) return sand::set_error(SAND_EINVAL, "rank >= world_size");
  for (uint32_t k = 0; k < s.n_views; ++k) {
    if (!out->data[k]) return sand::set_error(SAND_EINVAL, "null output pointer");
    if (reinterpret_cast<uintptr_t>(out->data[k]) % 16 != 0) return sand::set_error(SAND_EINVAL, "output not 16 B aligned");
  }
  auto stream = static_cast<cudaStream_t>(out->stream);
  std::unique_lock<std::mutex> lk(v->mu);
  auto plan = sand::get_plan(v, lk, epoch, rank);
  if (out->iteration >= plan->iterations) return sand::set_error(SAND_ERANGE, "iteration out of range");
  cudaError_t e = cudaSetDevice(v->store->device);
  if (e != cudaSuccess) return sand::cuda_error(e, "cudaSetDevice");
  if (!plan->uploaded) {
    int rc = sand::upload_plan(v, *plan, stream);
    if (rc != SAND_OK) return rc;
  }
  const uint64_t it = out->iteration;
  const uint32_t ib = plan->item_begin[it], ie = plan->item_begin[it + 1];
  // plan the next epoch on the worker while this one is consumed (pre-materialisation of the
  // plan, the analogue of the paper's pre-materialisation threads)
  if (it == 0) {
    const auto next = std::make_pair(epoch + 1, rank);
    if (!v->plans.count(next) && !v->pending.count(next)) {
      v->queue.push_back(next);
      v->cv.notify_all();
    }
  }
  sand_store* st = v->store;
  {
    std::lock_guard<std::mutex> slk(st->mu);
    for (uint32_t i = plan->fetch_begin[it]; i < plan->fetch_begin[it + 1]; ++i) {
      const auto& key = plan->fetch_keys[i];
      if (!st->videos.at(key.first).present[key.second])
        return sand::set_error(SAND_ENOENT, "frame " + std::to_string(key.second) + " of video " +
                                                std::to_string(key.first) + " is not in the store");
    }
  }
  sand::LaunchParams lp{};
  lp.slab = st->slab;
  lp.items = plan->d_items + ib;
  lp.n_items = ie - ib;
  lp.groups = plan->d_groups;
  lp.dests = plan->d_dests;
  lp.n_views = s.n_views;
  lp.batch = s.batch_size;
  for (uint32_t k = 0; k < s.n_views; ++k) {
    lp.out[k] = out->data[k];
    lp.views[k] = v->vconst[k];
  }
  int launched = 0;
  int rc = sand::launch_materialize(lp, plan->shapes[it], v->stencil_smem, stream, &launched);
  if (rc != SAND_OK) return rc;
  e = cudaEventRecord(plan->last_use, stream);
  if (e != cudaSuccess) return sand::cuda_error(e, "cudaEventRecord");
  {
    std::lock_guard<std::mutex> slk(st->mu);
    for (uint32_t i = plan->fetch_begin[it]; i < plan->fetch_begin[it + 1]; ++i) {
      auto& ve = st->videos.at(plan->fetch_keys[i].first);
      ve.fetches[plan->fetch_keys[i].second] += 1;
      ve.uses[plan->fetch_keys[i].second] += plan->fetch_uses[i];
    }
    st->batches++;
  }
  v->batches++;
  v->launches += static_cast<uint64_t>(launched);
  v->work_items += lp.n_items;
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
extern "C" int sand_view_batch_bytes(sand_view* v, uint64_t epoch, uint32_t rank, uint64_t iteration,
                                     sand_batch_bytes* out) {
  if (!v || !out) return sand::set_error(SAND_EINVAL, "null argument");
  if (rank >= v->info.spec.world_size) return sand::set_error(SAND_EINVAL, "rank >= world_size");
  std::unique_lock<std::mutex> lk(v->mu);
  auto plan = sand::get_plan(v, lk, epoch, rank);
  lk.unlock();
  if (iteration >= plan->iterations) return sand::set_error(SAND_ERANGE, "iteration out of range");
  const sand_view_spec& s = v->info.spec;
  std::memset(out, 0, sizeof(*out));
  for (uint32_t k = 0; k < s.n_views; ++k) {
    sand_tensor_desc td;
    sand_view_output_desc(v, k, &td);
    out->out_bytes += td.bytes;
  }
  // group items by source frame
  std::map<uint64_t, std::vector<uint32_t>> by_frame;
  for (uint32_t i = plan->item_begin[iteration]; i < plan->item_begin[iteration + 1]; ++i)
    by_frame[plan->items[i].y_off].push_back(i);
  for (auto& kv : by_frame) {
    const sand::WorkItem& w0 = plan->items[kv.second[0]];
    const uint32_t W = w0.src_w, H = w0.src_h, nsec = (W + 31) / 32;
    std::vector<uint8_t> ysec(static_cast<size_t>(H) * nsec, 0), uvsec(static_cast<size_t>(H / 2) * nsec, 0);
    for (uint32_t i : kv.second) {
      const sand::GroupParams& g = plan->groups[plan->items[i].gp];
      auto taps = [](float sc, int off, int n_out, int lim, int org, std::vector<uint8_t>& mark) {
        for (int o = 0; o < n_out; ++o) {
          const float sv = std::max(sc * (static_cast<float>(off + o) + 0.5f) - 0.5f, 0.0f);
          const int i0 = static_cast<int>(sv);
          const int i1 = std::min(i0 + 1, lim - 1);
          mark[org + i0] = 1;
          mark[org + i1] = 1;
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
  for (uint32_t i = plan->fetch_begin[iteration]; i < plan->fetch_begin[iteration + 1]; ++i) {
    out->fetches += 1;
    out->uses += plan->fetch_uses[i];
  }
  return SAND_OK;
}

extern "C" int sand_view_get_stats(const sand_view* v, sand_view_stats* out) {
  if (!v || !out) return sand::set_error(SAND_EINVAL, "null argument");
  out->batches = v->batches;
  out->kernel_launches = v->launches;
  out->plans_built = v->plans_built;
  out->work_items = v->work_items;
  return SAND_OK;
}

extern "C" int sand_view_destroy(sand_view* v) {
  if (!v) return SAND_OK;
  {
    std::lock_guard<std::mutex> lk(v->mu);
    v->stop = true;
    v->cv.notify_all();
  }
  if (v->worker.joinable()) v->worker.join();
  cudaSetDevice(v->store->device);
  for (auto& kv : v->plans) sand::release_plan_device(v, *kv.second);
  sand::free_pool(v);
  v->store->live_views--;
  delete v;
  return SAND_OK;
}
