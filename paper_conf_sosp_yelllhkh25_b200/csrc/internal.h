// internal.h — host runtime objects behind the C-ABI (store, view group, plans).
#pragma once
#include <cuda_runtime.h>

#include <atomic>
#include <condition_variable>
#include <cstdint>
#include <deque>
#include <map>
#include <memory>
#include <mutex>
#include <string>
#include <thread>
#include <unordered_map>
#include <vector>

#include "plan_types.h"
#include "planner.h"
#include "sand.h"

namespace sand {

// thread-local error message; every ABI function sets it before returning an error
int set_error(int code, const std::string& msg);
int cuda_error(cudaError_t e, const char* what);

// ------------------------------------------------------------------ HBM frame store (D4)
struct VideoEntry {
  uint32_t id, n_frames, width, height, pitch;
  uint64_t offset;         // slab offset of frame 0
  uint64_t frame_stride;   // bytes between frames
  std::vector<uint8_t> present;
  std::vector<uint64_t> fetches, uses;   // reuse accounting (a12)
};

}  // namespace sand

namespace sand {
// one frame of sand_store_put_frame_batch: source (packed buffer) and destination (slab) offsets
struct PutDesc {
  uint64_t src;       // byte offset of the frame's Y plane in the source buffer
  uint64_t dst;       // byte offset of the frame's slot in the slab
  uint32_t width, height, dst_pitch, pad;
};
// scatter n packed frames (Y rows then UV rows, source row pitch src_pitch, UV plane at
// src + uv_offset) into their slab slots with `word`-byte (16, 4 or 1) copies; stream-ordered
// (store_kernels.cu)
int launch_put_scatter(const uint8_t* src, uint64_t src_pitch, uint64_t uv_offset, uint8_t* slab,
                       const PutDesc* desc, uint32_t n, int word, cudaStream_t stream);
}  // namespace sand

struct sand_store {
  int device = 0;
  uint8_t* slab = nullptr;
  uint64_t capacity = 0, used = 0;
  std::unordered_map<uint32_t, sand::VideoEntry> videos;
  std::atomic<int> live_views{0};
  uint64_t batches = 0;
  std::mutex mu;   // guards counters updated by read_batch (views may live on several threads)
  // sand_store_put_frame_batch: device staging of packed host frames + per-frame descriptors,
  // reused across calls once `put_done` (recorded after the scatter) has completed
  uint8_t* put_stage = nullptr;
  uint64_t put_stage_bytes = 0;
  sand::PutDesc* put_desc = nullptr;        // device
  sand::PutDesc* put_desc_host = nullptr;   // pinned
  uint32_t put_desc_cap = 0;
  cudaEvent_t put_done = nullptr;
  // ordering of puts before reads: every put records `last_put` on its stream (after waiting on
  // the previous put's event, so puts on different streams are chained); read_batch makes its
  // stream wait on it whenever a put happened since that stream last waited
  cudaEvent_t last_put = nullptr;
  uint64_t put_seq = 0;
};

namespace sand {

// ------------------------------------------------------------------ epoch plan (D8)
struct EpochPlan {
  uint64_t epoch = 0;
  uint32_t rank = 0;
  uint64_t iterations = 0;
  std::vector<sand_clip_meta> metas;          // iterations * B
  std::vector<GroupParams> groups;            // iterations * B * n_groups
  std::vector<WorkItem> items;
  std::vector<uint32_t> dests;
  std::vector<uint2> tasks;                   // k_plain tasks (BatchShape::task_first / n_tasks)
  std::vector<uint32_t> item_begin;           // iterations + 1
  std::vector<BatchShape> shapes;             // per iteration: launch shape
  // reuse accounting per iteration: unique (video, frame) keys and their use counts
  std::vector<uint32_t> fetch_begin;          // iterations + 1
  std::vector<std::pair<uint32_t, uint32_t>> fetch_keys;   // (video, frame)
  std::vector<uint32_t> fetch_uses;
  std::vector<VideoEntry*> fetch_entry;       // store entry of each fetch key (stable: never erased)
  // device copy
  void* d_buf = nullptr;
  void* h_stage = nullptr;
  size_t d_bytes = 0;
  GroupParams* d_groups = nullptr;
  WorkItem* d_items = nullptr;
  uint32_t* d_dests = nullptr;
  uint2* d_tasks = nullptr;
  bool uploaded = false;
  cudaEvent_t last_use = nullptr;              // recorded after every kernel that reads the buffer
  cudaEvent_t ready = nullptr;                 // upload complete (recorded on the view's upload stream)
  cudaStream_t ready_waited = nullptr;         // last caller stream made to wait on `ready`
  uint64_t last_touch = 0;
  int pins = 0;                                // read_batch calls using the device copy (never evicted while > 0)
};

}  // namespace sand

namespace sand {
// A device + pinned-host buffer pair holding one uploaded epoch plan. Buffers of evicted plans
// are recycled instead of freed: cudaFree / cudaFreeHost synchronise the device and would stall
// the stream of read_batch calls at every epoch boundary.
struct PlanBuffer {
  void* d = nullptr;
  void* h = nullptr;
  size_t bytes = 0;
  cudaEvent_t done = nullptr;    // recorded after the last kernel that read the buffer
  cudaEvent_t ready = nullptr;   // recorded after the upload that wrote it
};
}  // namespace sand

struct sand_view {
  sand_store* store = nullptr;
  std::vector<sand::PlanBuffer> pool;   // recycled plan buffers (guarded by mu)
  sand::SpecInfo info;
  sand::ViewConst vconst[sand::kMaxViews];
  std::vector<uint32_t> video_slot;   // dataset index -> unused (dims live in info)
  // plan cache, keyed by (epoch, rank)
  std::mutex mu;
  std::condition_variable cv;
  std::map<std::pair<uint64_t, uint32_t>, std::shared_ptr<sand::EpochPlan>> plans;
  std::map<std::pair<uint64_t, uint32_t>, bool> pending;   // being built by the worker
  std::deque<std::pair<uint64_t, uint32_t>> queue;
  std::vector<std::thread> workers;     // plan builders (pre-materialisation threads)
  cudaStream_t upload_stream = nullptr;  // plan uploads (H2D), ordered before use by events
  std::vector<sand::VideoEntry*> entries;   // dataset index -> store entry (immutable geometry)
  std::vector<std::shared_ptr<sand::EpochPlan>> spare_plans;   // evicted plans, recycled by builders
  bool stop = false;
  uint64_t touch = 0;
  // stats
  uint64_t batches = 0, launches = 0, plans_built = 0, work_items = 0;
  uint64_t plan_build_ns = 0, plan_wait_ns = 0, read_ns = 0;
  uint64_t plan_cpu_ns = 0, plan_buffer_wait_ns = 0, lock_wait_ns = 0, pending_waits = 0;
  size_t stencil_smem = 0;   // dynamic smem of the stencil path (0 if no view rotates/blurs)
  int pl_fpc = 1, pl_nq = 1;     // k_plain: frames per CTA, threads per frame (from the widest view)
  size_t n_buffers = 0;          // plan buffers allocated so far
  std::vector<cudaEvent_t> inflight;   // ring of per-batch completion events (read-ahead bound)
  // batches with both direct and stencil items: the direct kernel runs on aux_stream (forked
  // from / joined to the caller's stream) so it fills the SMs the stencil kernel's tail leaves idle
  cudaStream_t aux_stream = nullptr;
  cudaEvent_t fork_ev = nullptr, join_ev = nullptr;
  // per-class kernel timing (sand_view_set_timing): event pairs recorded by read_batch
  bool timing = false;
  struct TimedLaunch {
    int cls;
    cudaEvent_t start, end;
  };
  std::vector<TimedLaunch> timed;                 // recorded, not yet collected
  std::vector<cudaEvent_t> free_events;
  double class_ms[3] = {0, 0, 0};
  uint64_t class_launches[3] = {0, 0, 0};
  // pre-materialisation (sand_view_prematerialize): batch buffers filled on a low-priority stream
  struct PreSlot {
    bool busy = false, acquired = false, consumed_pending = false;
    uint64_t epoch = 0, iteration = 0;
    uint32_t rank = 0;
    uint8_t* buf = nullptr;
    cudaEvent_t done = nullptr, consumed = nullptr;
  };
  std::vector<PreSlot> pre;
  size_t pre_view_off[sand::kMaxViews] = {};
  size_t pre_view_bytes[sand::kMaxViews] = {};
  cudaStream_t pre_stream = nullptr;
  uint64_t pre_made = 0, pre_served = 0;
  // HBM-budgeted object cache (f2, objcache.cpp): resized frames of short-side views
  uint64_t obj_budget = 0;
  struct ObjCache;
  ObjCache* obj = nullptr;
  uint64_t put_seq_seen = 0;              // store->put_seq the last read_batch stream waited for
  cudaStream_t put_stream_seen = nullptr;
};

namespace sand {

// Build the epoch plan of (epoch, rank) into `reuse` (a recycled plan whose device copy was
// released) or a new plan.
std::shared_ptr<EpochPlan> build_plan(const sand_view& v, uint64_t epoch, uint32_t rank,
                                      std::shared_ptr<EpochPlan> reuse = nullptr);
bool obj_eligible_group(const sand_view_spec& s, const SpecInfo& info, uint32_t q);
// launch shape of an arbitrary item list (view.cpp): classifies, orders (mild by clip/group/
// frame, heavy, stencil) and builds k_plain tasks, as build_plan does for a planned batch
void shape_items(const sand_view& v, std::vector<WorkItem>& items, const std::vector<GroupParams>& groups,
                 const std::vector<uint32_t>& dests, const ViewConst* views, uint32_t n_views, std::vector<uint2>* tasks,
                 BatchShape* shape);

// object cache (objcache.cpp, f2): one batch through the cache; *handled = false when the view
// has no cache (the caller then launches the plan's kernels)
int objcache_read(sand_view* v, EpochPlan& plan, uint64_t it, const LaunchParams& base, cudaStream_t stream,
                  int* launched, bool* handled);
int objcache_set_budget(sand_view* v, uint64_t bytes);
void objcache_free(sand_view* v);

// kernels (materialize.cu)
size_t stencil_smem_bytes(int max_h, int max_w, int max_r);
int configure_kernels(size_t stencil_smem);
// aux/fork/join may be null (then the kernels run back to back on `stream`)
// optional per-class event pairs recorded around each class's launch (null: no timing)
struct ClassEvents {
  cudaEvent_t start[3], end[3];
  bool used[3];
};
int launch_materialize(const LaunchParams& p, const BatchShape& shape, size_t stencil_smem, int pl_fpc, int pl_nq,
                       cudaStream_t stream, cudaStream_t aux, cudaEvent_t fork, cudaEvent_t join, int* n_launched,
                       ClassEvents* ev = nullptr);

}  // namespace sand
