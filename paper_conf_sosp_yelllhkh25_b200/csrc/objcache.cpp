// objcache.cpp — HBM-budgeted reuse of intermediate objects (§5.3
// Alg. 1 object-graph pruning, §6 eviction; R#27).
//
// The object is the RESIZED FRAME of a short-side view: the whole frame resized to W' x H'
// (uint8 R, G, B planes; Q2 at every crop position, R#10/R#12), keyed by (video, frame). All
// crops of a (video, frame) in any epoch of the k-epoch chunk and any view of the group are
// copies of it, bit-identical to resampling them from the NV12 frame.
//
// read_batch, per item of the batch in plan order (host, deterministic):
//   HIT   cached -> k_crop copies the crop from the object;
//   FILL  not cached; the object is used again in a later epoch of the chunk (Alg. 1: caching
//         the parent instead of its >= 2 leaves saves space, and the deterministic resize has no
//         randomness to preserve) and a slot is free after eviction -> the whole resized frame
//         is materialised into the slot by the ordinary kernels (a "virtual" uint8 view whose
//         tensor is the object slab), then k_crop copies the crop;
//   MISS  otherwise -> the item goes through the ordinary kernels.
// Eviction (§6: "When the storage usage exceeds 75 % of the designated threshold, SAND evicts
// (1) objects that have already been used and will not be required in future epochs, and (2)
// objects with the longest deadlines"): down to 75 % of the budget, when no slot is free for a
// fill (keeping the objects the current batch touched) and after every batch.
#include <cuda_runtime.h>

#include <algorithm>
#include <chrono>
#include <cstring>
#include <map>
#include <unordered_map>

#include "internal.h"
#include "kernels.h"

struct sand_view::ObjCache {
  uint8_t* slab = nullptr;
  uint64_t budget = 0, obj_bytes = 0;
  uint32_t n_slots = 0;
  uint32_t obj_w = 0, obj_h = 0, src_w = 0, src_h = 0;   // the one size class (set by the first object)
  std::vector<uint32_t> free_slots;
  struct Obj {
    uint32_t slot;
    uint32_t remaining;      // later uses in the chunk of its last touch
    uint64_t chunk;          // k-epoch chunk of its last touch
    uint64_t next_epoch;     // next planned use (UINT64_MAX: none)
    uint64_t last_batch;     // batch sequence number of its last touch (LRU)
  };
  std::unordered_map<uint64_t, Obj> objs;   // key: video id << 32 | frame
  uint64_t seq = 0;
  sand_object_stats stats{};
  // per-batch device arrays (fills, crops, misses), a small ring guarded by events
  struct Stage {
    void* d = nullptr;
    void* h = nullptr;
    size_t bytes = 0;
    cudaEvent_t done = nullptr;
    bool used = false;
  };
  Stage ring[4];
  size_t ring_pos = 0;
  cudaEvent_t batch_done = nullptr;
  bool batch_recorded = false;
};

namespace sand {

namespace {
size_t a256(size_t x) { return (x + 255) / 256 * 256; }
uint64_t now_ns() {
  return static_cast<uint64_t>(
      std::chrono::duration_cast<std::chrono::nanoseconds>(std::chrono::steady_clock::now().time_since_epoch()).count());
}
}  // namespace

void objcache_free(sand_view* v) {
  if (!v->obj) return;
  auto* c = v->obj;
  for (auto& st : c->ring) {
    if (st.done) {
      cudaEventSynchronize(st.done);
      cudaEventDestroy(st.done);
    }
    cudaFree(st.d);
    cudaFreeHost(st.h);
  }
  if (c->batch_done) {
    cudaEventSynchronize(c->batch_done);
    cudaEventDestroy(c->batch_done);
  }
  cudaFree(c->slab);
  delete c;
  v->obj = nullptr;
}

int objcache_set_budget(sand_view* v, uint64_t bytes) {
  objcache_free(v);
  v->obj_budget = bytes;
  if (bytes == 0) return SAND_OK;
  const sand_view_spec& s = v->info.spec;
  if (s.n_views >= kMaxViews) return set_error(SAND_EINVAL, "object cache needs a free view slot");
  for (uint32_t k = 1; k < s.n_views; ++k)
    if (s.views[k].out_dtype != s.views[0].out_dtype) return set_error(SAND_EINVAL, "object cache needs one output dtype");
  auto* c = new sand_view::ObjCache();
  c->budget = bytes;
  cudaError_t e = cudaMalloc(&c->slab, bytes);
  if (e == cudaSuccess) e = cudaEventCreateWithFlags(&c->batch_done, cudaEventDisableTiming);
  for (auto& st : c->ring)
    if (e == cudaSuccess) e = cudaEventCreateWithFlags(&st.done, cudaEventDisableTiming);
  v->obj = c;
  if (e != cudaSuccess) {
    objcache_free(v);
    v->obj_budget = 0;
    return cuda_error(e, "object cache allocation");
  }
  return SAND_OK;
}

namespace {

// §6 eviction down to 75 % of the budget: candidates ordered (1) not needed again in the current
// chunk, least recently used first, then (2) by the latest next use (ties: least recently used,
// then key); during a batch its own objects are kept (protect_batch). Returns objects evicted.
size_t evict_to_threshold(sand_view::ObjCache* c, uint64_t epoch, uint64_t chunk, bool protect_batch) {
  const uint64_t keep = c->budget * 3 / (4 * c->obj_bytes);     // objects allowed at 75 %
  if (c->objs.size() <= keep) return 0;
  struct Cand {
    int needed;
    uint64_t k1, k2, key;
    bool operator<(const Cand& b) const {
      if (needed != b.needed) return needed < b.needed;
      if (k1 != b.k1) return k1 < b.k1;
      if (k2 != b.k2) return k2 < b.k2;
      return key < b.key;
    }
  };
  std::vector<Cand> cand;
  cand.reserve(c->objs.size());
  for (const auto& kv : c->objs) {
    const auto& o = kv.second;
    if (protect_batch && o.last_batch == c->seq) continue;
    const bool needed = o.remaining > 0 && o.chunk == chunk && o.next_epoch != UINT64_MAX && o.next_epoch >= epoch;
    if (needed) cand.push_back({1, ~o.next_epoch, o.last_batch, kv.first});
    else cand.push_back({0, o.last_batch, 0, kv.first});
  }
  const size_t n = std::min<size_t>(cand.size(), c->objs.size() - keep);
  std::partial_sort(cand.begin(), cand.begin() + n, cand.end());   // the n first victims, in order
  for (size_t i = 0; i < n; ++i) {
    auto it = c->objs.find(cand[i].key);
    c->free_slots.push_back(it->second.slot);
    c->objs.erase(it);
  }
  c->stats.evictions += n;
  return n;
}

template <typename T>
size_t put(std::vector<uint8_t>& buf, const std::vector<T>& v) {
  const size_t off = a256(buf.size());
  buf.resize(off + v.size() * sizeof(T));
  if (!v.empty()) std::memcpy(buf.data() + off, v.data(), v.size() * sizeof(T));
  return off;
}

}  // namespace

int objcache_read(sand_view* v, EpochPlan& plan, uint64_t it, const LaunchParams& base, cudaStream_t stream,
                  int* launched, bool* handled) {
  *handled = false;
  *launched = 0;
  auto* c = v->obj;
  if (!c) return SAND_OK;
  *handled = true;
  const uint64_t t0 = now_ns();
  const sand_view_spec& s = v->info.spec;
  const uint32_t B = s.batch_size;
  const uint32_t kch = std::max<uint32_t>(1, s.pool_epochs);
  const uint64_t epoch = plan.epoch, chunk = epoch / kch;
  const uint32_t vview = s.n_views;
  c->seq++;
  std::vector<WorkItem> fills, misses;
  std::vector<uint32_t> fill_dests;
  std::vector<CropItem> crops;
  int32_t crop_wo = 0, crop_ho = 0;
  // items in canonical order (clip slot, frame, group): the decisions below do not depend on
  // how the plan ordered its items for the kernels
  const uint32_t ib = plan.item_begin[it], ie = plan.item_begin[it + 1];
  std::vector<uint32_t> order(ie - ib);
  for (uint32_t i = ib; i < ie; ++i) order[i - ib] = i;
  std::sort(order.begin(), order.end(), [&](uint32_t a, uint32_t b) {
    const WorkItem &x = plan.items[a], &y = plan.items[b];
    if (x.clip_slot != y.clip_slot) return x.clip_slot < y.clip_slot;
    if (x.y_off != y.y_off) return x.y_off < y.y_off;
    return x.group < y.group;
  });
  for (uint32_t i : order) {
    const WorkItem& w = plan.items[i];
    const sand_clip_meta& m = plan.metas[it * B + w.clip_slot];
    bool eligible = !(w.flags & 1u) && obj_eligible_group(s, v->info, w.group);
    const int32_t* box = m.box[w.group];
    if (eligible && c->obj_w == 0) {      // the first object fixes the size class and the slots
      c->obj_w = static_cast<uint32_t>(box[2]);
      c->obj_h = static_cast<uint32_t>(box[3]);
      c->src_w = w.src_w;
      c->src_h = w.src_h;
      // object b of the virtual view sits at b * 3 W' H' (its tensor layout); 16 B of slack at the
      // end of the slab for the crop kernel's aligned over-read
      c->obj_bytes = 3ull * c->obj_w * c->obj_h;
      c->n_slots = static_cast<uint32_t>(std::min<uint64_t>(c->budget > 16 ? (c->budget - 16) / c->obj_bytes : 0, 65535));
      for (uint32_t k = c->n_slots; k-- > 0;) c->free_slots.push_back(k);
      c->stats.bytes_budget = c->budget;
    }
    eligible = eligible && static_cast<uint32_t>(box[2]) == c->obj_w && static_cast<uint32_t>(box[3]) == c->obj_h &&
               w.src_w == c->src_w && w.src_h == c->src_h;
    if (!eligible) {
      misses.push_back(w);
      continue;
    }
    const VideoEntry* ent = v->entries[m.clip / s.samples_per_video];
    const uint32_t frame = static_cast<uint32_t>((w.y_off - ent->offset) / ent->frame_stride);
    const uint64_t key = (static_cast<uint64_t>(ent->id) << 32) | frame;
    const uint32_t later = w.pad >> 16, next_delta = w.pad & 0xffffu;
    auto found = c->objs.find(key);
    bool cached = found != c->objs.end();
    if (!cached && later >= 1) {          // FILL: worth caching (reused later in the chunk)
      if (c->free_slots.empty()) evict_to_threshold(c, epoch, chunk, true);
      if (!c->free_slots.empty()) {
        sand_view::ObjCache::Obj o{};
        o.slot = c->free_slots.back();
        c->free_slots.pop_back();
        WorkItem f = w;
        f.gp = 0;                          // the resize geometry (fill group 0)
        f.dest_begin = static_cast<uint32_t>(fill_dests.size());
        f.n_dest = 1;
        f.group = 0;
        f.flags = 0;
        fill_dests.push_back(pack_dest(vview, 0, o.slot));
        fills.push_back(f);
        found = c->objs.emplace(key, o).first;
        cached = true;
        c->stats.fills++;
      }
    } else if (cached) {
      c->stats.hits++;
    }
    if (!cached) {
      c->stats.misses++;
      misses.push_back(w);
      continue;
    }
    auto& o = found->second;
    o.remaining = later;
    o.chunk = chunk;
    o.next_epoch = next_delta == 0xffffu ? UINT64_MAX : epoch + next_delta;
    o.last_batch = c->seq;
    const GroupParams& g = plan.groups[w.gp];
    CropItem ci{};
    ci.obj = static_cast<uint64_t>(o.slot) * c->obj_bytes;
    ci.obj_w = c->obj_w;
    ci.obj_h = c->obj_h;
    ci.x_off = static_cast<uint32_t>(box[0]);
    ci.y_off = static_cast<uint32_t>(box[1]);
    ci.flip = static_cast<uint32_t>(g.flip);
    ci.out_w = static_cast<uint32_t>(g.out_w);
    ci.out_h = static_cast<uint32_t>(g.out_h);
    ci.dest_begin = w.dest_begin;
    ci.n_dest = w.n_dest;
    crops.push_back(ci);
    crop_wo = std::max(crop_wo, g.out_w);
    crop_ho = std::max(crop_ho, g.out_h);
  }
  // after the batch (its crops are stream-ordered before any later fill): keep usage at or
  // below 75 % of the budget (§6)
  auto used = [&]() { return static_cast<uint64_t>(c->objs.size()) * c->obj_bytes; };
  evict_to_threshold(c, epoch, chunk, false);
  c->stats.objects = c->objs.size();
  c->stats.bytes_used = used();

  // shapes and tasks of the fill and miss lists
  std::vector<GroupParams> fill_groups;
  ViewConst views[kMaxViews];
  std::memcpy(views, base.views, sizeof(views));
  if (!fills.empty()) {
    GroupParams g{};
    g.lim_x = static_cast<int32_t>(c->src_w);
    g.lim_y = static_cast<int32_t>(c->src_h);
    g.out_w = static_cast<int32_t>(c->obj_w);
    g.out_h = static_cast<int32_t>(c->obj_h);
    g.sc_x = static_cast<float>(c->src_w) / static_cast<float>(c->obj_w);   // as group_params (view.cpp)
    g.sc_y = static_cast<float>(c->src_h) / static_cast<float>(c->obj_h);
    fill_groups.push_back(g);
    ViewConst& vc = views[vview];
    vc = ViewConst{};
    vc.dtype = SAND_U8;
    vc.T = 1;
    vc.out_h = static_cast<int32_t>(c->obj_h);
    vc.out_w = static_cast<int32_t>(c->obj_w);
  }
  std::vector<uint2> fill_tasks, miss_tasks;
  BatchShape fill_shape{}, miss_shape{};
  if (!fills.empty()) shape_items(*v, fills, fill_groups, fill_dests, views, vview + 1, &fill_tasks, &fill_shape);
  if (!misses.empty()) shape_items(*v, misses, plan.groups, plan.dests, base.views, s.n_views, &miss_tasks, &miss_shape);

  const uint64_t t1 = now_ns();
  // stage the per-batch arrays (one H2D copy on the caller's stream)
  std::vector<uint8_t> hbuf;
  const size_t o_fg = put(hbuf, fill_groups), o_fi = put(hbuf, fills), o_fd = put(hbuf, fill_dests),
               o_ft = put(hbuf, fill_tasks), o_ci = put(hbuf, crops), o_mi = put(hbuf, misses), o_mt = put(hbuf, miss_tasks);
  auto& st = c->ring[c->ring_pos];
  c->ring_pos = (c->ring_pos + 1) % 4;
  cudaError_t e = cudaSuccess;
  if (st.used) e = cudaEventSynchronize(st.done);   // its previous batch's kernels are done
  if (e == cudaSuccess && st.bytes < hbuf.size() + 256) {
    cudaFree(st.d);
    cudaFreeHost(st.h);
    st.d = st.h = nullptr;
    st.bytes = a256(hbuf.size() + hbuf.size() / 2 + 4096);
    e = cudaMalloc(&st.d, st.bytes);
    if (e == cudaSuccess) e = cudaMallocHost(&st.h, st.bytes);
  }
  if (e != cudaSuccess) return cuda_error(e, "object cache staging");
  if (!hbuf.empty()) std::memcpy(st.h, hbuf.data(), hbuf.size());
  if (c->batch_recorded) e = cudaStreamWaitEvent(stream, c->batch_done, 0);   // object slots of the last batch
  if (e == cudaSuccess && !hbuf.empty()) e = cudaMemcpyAsync(st.d, st.h, hbuf.size(), cudaMemcpyHostToDevice, stream);
  if (e != cudaSuccess) return cuda_error(e, "object cache staging copy");
  auto* d = static_cast<uint8_t*>(st.d);
  const uint64_t t2 = now_ns();

  int n = 0, rc = SAND_OK;
  if (!fills.empty()) {                 // resized frames into their slots (a uint8 virtual view)
    LaunchParams pf = base;
    pf.items = reinterpret_cast<const WorkItem*>(d + o_fi);
    pf.n_items = static_cast<uint32_t>(fills.size());
    pf.groups = reinterpret_cast<const GroupParams*>(d + o_fg);
    pf.dests = reinterpret_cast<const uint32_t*>(d + o_fd);
    pf.tasks = reinterpret_cast<const uint2*>(d + o_ft);
    pf.views[vview] = views[vview];
    pf.out[vview] = c->slab;
    pf.n_views = vview + 1;
    int k = 0;
    rc = launch_materialize(pf, fill_shape, v->stencil_smem, v->pl_fpc, v->pl_nq, stream, nullptr, nullptr, nullptr, &k);
    n += k;
  }
  if (rc == SAND_OK && !crops.empty()) {
    rc = launch_crop(base, c->slab, d + o_ci, static_cast<uint32_t>(crops.size()), crop_wo, crop_ho,
                     s.views[0].out_dtype, stream);
    n += 1;
  }
  if (rc == SAND_OK && !misses.empty()) {
    LaunchParams pm = base;
    pm.items = reinterpret_cast<const WorkItem*>(d + o_mi);
    pm.n_items = static_cast<uint32_t>(misses.size());
    pm.tasks = reinterpret_cast<const uint2*>(d + o_mt);
    int k = 0;
    rc = launch_materialize(pm, miss_shape, v->stencil_smem, v->pl_fpc, v->pl_nq, stream, v->aux_stream, v->fork_ev,
                            v->join_ev, &k);
    n += k;
  }
  if (rc != SAND_OK) return rc;
  e = cudaEventRecord(st.done, stream);
  if (e == cudaSuccess) e = cudaEventRecord(c->batch_done, stream);
  if (e != cudaSuccess) return cuda_error(e, "object cache events");
  st.used = true;
  c->batch_recorded = true;
  *launched = n;
  const uint64_t t3 = now_ns();
  c->stats.decide_ns += t1 - t0;
  c->stats.stage_ns += t2 - t1;
  c->stats.launch_ns += t3 - t2;
  return SAND_OK;
}

}  // namespace sand

extern "C" int sand_view_set_object_budget(sand_view* v, uint64_t bytes) {
  if (!v) return sand::set_error(SAND_EINVAL, "null argument");
  std::unique_lock<std::mutex> lk(v->mu);
  // plans carry the later-use counts (WorkItem.pad) only when a budget is set: it must be set
  // before the view plans anything
  if (!v->plans.empty() || !v->pending.empty() || !v->queue.empty() || v->batches > 0)
    return sand::set_error(SAND_EBUSY, "set the object budget before the view plans or reads");
  cudaError_t e = cudaSetDevice(v->store->device);
  if (e != cudaSuccess) return sand::cuda_error(e, "cudaSetDevice");
  return sand::objcache_set_budget(v, bytes);
}

extern "C" int sand_view_object_stats(const sand_view* v, sand_object_stats* out) {
  if (!v || !out) return sand::set_error(SAND_EINVAL, "null argument");
  std::memset(out, 0, sizeof(*out));
  if (v->obj) *out = v->obj->stats;
  out->bytes_budget = v->obj_budget;
  return SAND_OK;
}
