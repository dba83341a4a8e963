// store.cpp — the HBM decoded-frame store keyed by (video, frame) with reuse
// accounting. SAND keeps decoded uint8 frames as objects in
// memory or storage (§6); here every frame of the dataset is resident in
// one pitched device slab, NV12, row pitch a multiple of 64 B.
#include <cuda_runtime.h>

#include <algorithm>
#include <cstring>

#include "internal.h"

using sand::VideoEntry;

namespace {
constexpr uint64_t kPitchAlign = 64;
constexpr uint64_t kFrameAlign = 256;
uint64_t align_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }
}  // namespace

extern "C" int sand_store_create(int cuda_device, uint64_t capacity_bytes, sand_store** out) {
  if (!out) return sand::set_error(SAND_EINVAL, "out is null");
  *out = nullptr;
  if (capacity_bytes == 0) return sand::set_error(SAND_EINVAL, "capacity must be > 0");
  int n = 0;
  cudaError_t e = cudaGetDeviceCount(&n);
  if (e != cudaSuccess) return sand::cuda_error(e, "cudaGetDeviceCount");
  if (cuda_device < 0 || cuda_device >= n) return sand::set_error(SAND_EINVAL, "bad cuda_device");
  if ((e = cudaSetDevice(cuda_device)) != cudaSuccess) return sand::cuda_error(e, "cudaSetDevice");
  auto* s = new sand_store();
  s->device = cuda_device;
  s->capacity = align_up(capacity_bytes, kFrameAlign);
  e = cudaMalloc(reinterpret_cast<void**>(&s->slab), s->capacity);
  if (e != cudaSuccess) {
    delete s;
    cudaGetLastError();
    return sand::set_error(SAND_ENOMEM, std::string("cudaMalloc of the frame slab failed: ") + cudaGetErrorString(e));
  }
  *out = s;
  return SAND_OK;
}

extern "C" int sand_store_add_video(sand_store* s, uint32_t video, uint32_t n_frames, uint32_t width,
                                    uint32_t height) {
  if (!s) return sand::set_error(SAND_EINVAL, "store is null");
  if (width == 0 || height == 0 || (width & 1u) || (height & 1u) || n_frames == 0)
    return sand::set_error(SAND_EINVAL, "NV12 frames need even, non-zero width/height and n_frames > 0");
  if (width > 4096 || height > 4096) return sand::set_error(SAND_EINVAL, "frames larger than 4096x4096");
  std::lock_guard<std::mutex> lk(s->mu);
  auto it = s->videos.find(video);
  if (it != s->videos.end()) {
    const VideoEntry& v = it->second;
    if (v.n_frames == n_frames && v.width == width && v.height == height) return SAND_OK;
    return sand::set_error(SAND_EINVAL, "video already added with different dimensions");
  }
  VideoEntry v;
  v.id = video;
  v.n_frames = n_frames;
  v.width = width;
  v.height = height;
  v.pitch = static_cast<uint32_t>(align_up(width, kPitchAlign));
  v.frame_stride = align_up(static_cast<uint64_t>(v.pitch) * (height + height / 2), kFrameAlign);
  const uint64_t need = v.frame_stride * n_frames;
  if (s->used + need > s->capacity) return sand::set_error(SAND_ENOMEM, "frame store capacity exceeded");
  v.offset = s->used;
  s->used += need;
  v.present.assign(n_frames, 0);
  v.fetches.assign(n_frames, 0);
  v.uses.assign(n_frames, 0);
  s->videos.emplace(video, std::move(v));
  return SAND_OK;
}

namespace {
// order a put on `st` after the previous put (any stream); call before enqueuing its copies
int put_begin(sand_store* s, cudaStream_t st) {
  if (!s->last_put) {
    cudaError_t e = cudaEventCreateWithFlags(&s->last_put, cudaEventDisableTiming);
    if (e != cudaSuccess) return sand::cuda_error(e, "cudaEventCreate(last_put)");
  } else if (s->put_seq > 0) {
    cudaError_t e = cudaStreamWaitEvent(st, s->last_put, 0);
    if (e != cudaSuccess) return sand::cuda_error(e, "cudaStreamWaitEvent(last_put)");
  }
  return SAND_OK;
}
int put_end(sand_store* s, cudaStream_t st) {
  cudaError_t e = cudaEventRecord(s->last_put, st);
  if (e != cudaSuccess) return sand::cuda_error(e, "cudaEventRecord(last_put)");
  s->put_seq++;
  return SAND_OK;
}
}  // namespace

extern "C" int sand_store_put_frames(sand_store* s, uint32_t video, uint32_t first_frame, uint32_t n_frames,
                                     const uint8_t* y, uint64_t y_pitch, uint64_t y_frame_stride,
                                     const uint8_t* uv, uint64_t uv_pitch, uint64_t uv_frame_stride,
                                     int src_on_device, sand_stream_t stream) {
  if (!s || !y || !uv) return sand::set_error(SAND_EINVAL, "null argument");
  std::lock_guard<std::mutex> lk(s->mu);
  auto it = s->videos.find(video);
  if (it == s->videos.end()) return sand::set_error(SAND_ERANGE, "unknown video (call sand_store_add_video)");
  VideoEntry& v = it->second;
  if (static_cast<uint64_t>(first_frame) + n_frames > v.n_frames)
    return sand::set_error(SAND_ERANGE, "frame range outside the video");
  if (y_pitch < v.width || uv_pitch < v.width) return sand::set_error(SAND_EINVAL, "pitch < width");
  cudaError_t e = cudaSetDevice(s->device);
  if (e != cudaSuccess) return sand::cuda_error(e, "cudaSetDevice");
  const cudaMemcpyKind kind = src_on_device ? cudaMemcpyDeviceToDevice : cudaMemcpyHostToDevice;
  auto st = static_cast<cudaStream_t>(stream);
  int rc = put_begin(s, st);
  if (rc != SAND_OK) return rc;
  for (uint32_t f = 0; f < n_frames; ++f) {
    uint8_t* dst = s->slab + v.offset + v.frame_stride * (first_frame + f);
    e = cudaMemcpy2DAsync(dst, v.pitch, y + y_frame_stride * f, y_pitch, v.width, v.height, kind, st);
    if (e != cudaSuccess) return sand::cuda_error(e, "cudaMemcpy2DAsync(Y)");
    e = cudaMemcpy2DAsync(dst + static_cast<uint64_t>(v.pitch) * v.height, v.pitch, uv + uv_frame_stride * f,
                          uv_pitch, v.width, v.height / 2, kind, st);
    if (e != cudaSuccess) return sand::cuda_error(e, "cudaMemcpy2DAsync(UV)");
    v.present[first_frame + f] = 1;
    v.fetches[first_frame + f] = 0;
    v.uses[first_frame + f] = 0;
  }
  return put_end(s, st);
}

extern "C" int sand_store_put_frame_batch(sand_store* s, uint32_t n, const uint32_t* videos, const uint32_t* frames,
                                          const uint8_t* src, uint64_t frame_stride, uint64_t pitch,
                                          uint64_t uv_offset, int src_on_device, sand_stream_t stream) {
  if (!s || (n > 0 && (!videos || !frames || !src))) return sand::set_error(SAND_EINVAL, "null argument");
  if (n == 0) return SAND_OK;
  std::lock_guard<std::mutex> lk(s->mu);
  // validate every (video, frame) first: nothing is copied on error
  uint32_t width = 0, height = 0;
  for (uint32_t i = 0; i < n; ++i) {
    auto it = s->videos.find(videos[i]);
    if (it == s->videos.end() || frames[i] >= it->second.n_frames)
      return sand::set_error(SAND_ERANGE, "unknown (video, frame) in batch put");
    const VideoEntry& v = it->second;
    if (i == 0) {
      width = v.width;
      height = v.height;
    } else if (v.width != width || v.height != height) {
      return sand::set_error(SAND_EINVAL, "batch put frames must share width and height");
    }
  }
  if (pitch < width || uv_offset < pitch * height || frame_stride < uv_offset + pitch * (height / 2 - 1) + width)
    return sand::set_error(SAND_EINVAL, "pitch / uv_offset / frame_stride do not fit the frames");
  cudaError_t e = cudaSetDevice(s->device);
  if (e != cudaSuccess) return sand::cuda_error(e, "cudaSetDevice");
  auto st = static_cast<cudaStream_t>(stream);
  if (!s->put_done) {
    e = cudaEventCreateWithFlags(&s->put_done, cudaEventDisableTiming);
    if (e != cudaSuccess) return sand::cuda_error(e, "cudaEventCreate(put_done)");
  }
  // the staging buffers of the previous call are reusable once its scatter has run
  e = cudaEventSynchronize(s->put_done);
  if (e != cudaSuccess) return sand::cuda_error(e, "cudaEventSynchronize(put_done)");
  {
    const int prc = put_begin(s, st);
    if (prc != SAND_OK) return prc;
  }
  if (s->put_desc_cap < n) {
    cudaFree(s->put_desc);
    cudaFreeHost(s->put_desc_host);
    s->put_desc = nullptr;
    s->put_desc_host = nullptr;
    s->put_desc_cap = 0;
    const uint32_t cap = std::max<uint32_t>(n, 1024);
    e = cudaMalloc(reinterpret_cast<void**>(&s->put_desc), sizeof(sand::PutDesc) * cap);
    if (e == cudaSuccess) e = cudaMallocHost(reinterpret_cast<void**>(&s->put_desc_host), sizeof(sand::PutDesc) * cap);
    if (e != cudaSuccess) return sand::cuda_error(e, "batch put descriptor buffers");
    s->put_desc_cap = cap;
  }
  const uint64_t bytes = frame_stride * (n - 1) + uv_offset + pitch * (height / 2 - 1) + width;
  const uint8_t* dsrc = src;
  if (!src_on_device) {                  // one host->device transfer of the whole packed batch
    if (s->put_stage_bytes < bytes) {
      cudaFree(s->put_stage);
      s->put_stage = nullptr;
      s->put_stage_bytes = 0;
      e = cudaMalloc(reinterpret_cast<void**>(&s->put_stage), bytes);
      if (e != cudaSuccess) return sand::cuda_error(e, "batch put staging buffer");
      s->put_stage_bytes = bytes;
    }
    e = cudaMemcpyAsync(s->put_stage, src, bytes, cudaMemcpyHostToDevice, st);
    if (e != cudaSuccess) return sand::cuda_error(e, "cudaMemcpyAsync(batch put)");
    dsrc = s->put_stage;
  }
  for (uint32_t i = 0; i < n; ++i) {
    VideoEntry& v = s->videos.find(videos[i])->second;
    sand::PutDesc& d = s->put_desc_host[i];
    d.src = frame_stride * i;
    d.dst = v.offset + v.frame_stride * frames[i];
    d.width = v.width;
    d.height = v.height;
    d.dst_pitch = v.pitch;
    d.pad = 0;
    v.present[frames[i]] = 1;
    v.fetches[frames[i]] = 0;
    v.uses[frames[i]] = 0;
  }
  e = cudaMemcpyAsync(s->put_desc, s->put_desc_host, sizeof(sand::PutDesc) * n, cudaMemcpyHostToDevice, st);
  if (e != cudaSuccess) return sand::cuda_error(e, "cudaMemcpyAsync(batch put descriptors)");
  // widest copy word every row start allows (slab rows are 64 B aligned)
  const uint64_t al = reinterpret_cast<uintptr_t>(dsrc) | frame_stride | pitch | uv_offset | width;
  const int word = (al & 15) == 0 ? 16 : ((al & 3) == 0 ? 4 : 1);
  const int rc = sand::launch_put_scatter(dsrc, pitch, uv_offset, s->slab, s->put_desc, n, word, st);
  if (rc != SAND_OK) return rc;
  e = cudaEventRecord(s->put_done, st);
  if (e != cudaSuccess) return sand::cuda_error(e, "cudaEventRecord(put_done)");
  return put_end(s, st);
}

extern "C" int sand_store_frame_layout(const sand_store* s, uint32_t video, uint32_t frame,
                                       sand_frame_layout* out) {
  if (!s || !out) return sand::set_error(SAND_EINVAL, "null argument");
  auto it = s->videos.find(video);
  if (it == s->videos.end() || frame >= it->second.n_frames)
    return sand::set_error(SAND_ERANGE, "unknown (video, frame)");
  const VideoEntry& v = it->second;
  const uint64_t base = reinterpret_cast<uint64_t>(s->slab) + v.offset + v.frame_stride * frame;
  out->y = base;
  out->uv = base + static_cast<uint64_t>(v.pitch) * v.height;
  out->pitch = v.pitch;
  out->width = v.width;
  out->height = v.height;
  out->n_frames = v.n_frames;
  out->frame_stride = v.frame_stride;
  return SAND_OK;
}

extern "C" int sand_store_mark_present(sand_store* s, uint32_t video, uint32_t first_frame, uint32_t n_frames) {
  if (!s) return sand::set_error(SAND_EINVAL, "store is null");
  std::lock_guard<std::mutex> lk(s->mu);
  auto it = s->videos.find(video);
  if (it == s->videos.end() || static_cast<uint64_t>(first_frame) + n_frames > it->second.n_frames)
    return sand::set_error(SAND_ERANGE, "unknown (video, frame range)");
  for (uint32_t f = first_frame; f < first_frame + n_frames; ++f) {
    it->second.present[f] = 1;
    it->second.fetches[f] = 0;
    it->second.uses[f] = 0;
  }
  return SAND_OK;
}

extern "C" int sand_store_counters(const sand_store* s, sand_counters* out) {
  if (!s || !out) return sand::set_error(SAND_EINVAL, "null argument");
  auto* ms = const_cast<sand_store*>(s);
  std::lock_guard<std::mutex> lk(ms->mu);
  std::memset(out, 0, sizeof(*out));
  out->videos = s->videos.size();
  out->bytes_reserved = s->used;
  out->capacity = s->capacity;
  out->batches = s->batches;
  for (const auto& kv : s->videos) {
    for (uint32_t f = 0; f < kv.second.n_frames; ++f) {
      out->frames_present += kv.second.present[f];
      out->fetches += kv.second.fetches[f];
      out->uses += kv.second.uses[f];
    }
  }
  return SAND_OK;
}

extern "C" int sand_store_frame_counters(const sand_store* s, uint32_t video, uint32_t first, uint32_t n,
                                         uint64_t* fetches, uint64_t* uses) {
  if (!s) return sand::set_error(SAND_EINVAL, "store is null");
  auto* ms = const_cast<sand_store*>(s);
  std::lock_guard<std::mutex> lk(ms->mu);
  auto it = s->videos.find(video);
  if (it == s->videos.end() || static_cast<uint64_t>(first) + n > it->second.n_frames)
    return sand::set_error(SAND_ERANGE, "unknown (video, frame range)");
  for (uint32_t i = 0; i < n; ++i) {
    if (fetches) fetches[i] = it->second.fetches[first + i];
    if (uses) uses[i] = it->second.uses[first + i];
  }
  return SAND_OK;
}

extern "C" int sand_store_destroy(sand_store* s) {
  if (!s) return SAND_OK;
  if (s->live_views.load() > 0) return sand::set_error(SAND_EBUSY, "store has live views");
  cudaSetDevice(s->device);
  cudaDeviceSynchronize();
  cudaFree(s->slab);
  cudaFree(s->put_stage);
  cudaFree(s->put_desc);
  cudaFreeHost(s->put_desc_host);
  if (s->put_done) cudaEventDestroy(s->put_done);
  if (s->last_put) cudaEventDestroy(s->last_put);
  delete s;
  return SAND_OK;
}
