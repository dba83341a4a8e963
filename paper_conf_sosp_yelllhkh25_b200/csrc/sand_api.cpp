// sand_api.cpp — error reporting and version of the C-ABI (include/sand.h).
#include <cuda_runtime.h>

#include <algorithm>
#include <string>

#include "internal.h"

namespace sand {
namespace {
thread_local std::string g_last_error;
}

int set_error(int code, const std::string& msg) {
  g_last_error = msg;
  return code;
}

int cuda_error(cudaError_t e, const char* what) {
  g_last_error = std::string(what) + ": " + cudaGetErrorString(e);
  cudaGetLastError();   // clear the sticky-free error state
  return SAND_ECUDA;
}

}  // namespace sand

extern "C" const char* sand_last_error(void) { return sand::g_last_error.c_str(); }

extern "C" const char* sand_version(void) { return "sand-b200 0.1 (sm_100a)"; }

extern "C" int sand_abi_sizes(uint64_t sizes[8]) {
  if (!sizes) return sand::set_error(SAND_EINVAL, "null argument");
  sizes[0] = sizeof(sand_frame_layout);
  sizes[1] = sizeof(sand_counters);
  sizes[2] = sizeof(sand_view_desc);
  sizes[3] = sizeof(sand_view_spec);
  sizes[4] = sizeof(sand_tensor_desc);
  sizes[5] = sizeof(sand_batch_out);
  sizes[6] = sizeof(sand_clip_meta);
  sizes[7] = sizeof(sand_batch_bytes);
  return 8;
}

namespace {
int host_spec(const sand_view_spec* spec, const uint32_t* n_frames, const uint32_t* widths, const uint32_t* heights,
              sand::SpecInfo* info) {
  if (!spec) return sand::set_error(SAND_EINVAL, "null spec");
  std::string why;
  const int rc = sand::validate_spec(*spec, &why);
  if (rc != SAND_OK) return sand::set_error(rc, why);
  info->spec = *spec;
  info->videos.assign(spec->videos, spec->videos + spec->n_videos);
  info->spec.videos = info->videos.data();
  for (uint32_t i = 0; i < spec->n_videos; ++i)
    info->dims.push_back({spec->videos[i], n_frames ? n_frames[i] : 1u, widths ? widths[i] : 2u,
                          heights ? heights[i] : 2u});
  sand::derive_spec(info);
  return SAND_OK;
}
}  // namespace

extern "C" int sand_plan_rank_clips(const sand_view_spec* spec, uint64_t epoch, uint32_t rank, uint32_t* out,
                                    uint32_t cap, uint32_t* n) {
  if (!out || !n) return sand::set_error(SAND_EINVAL, "null argument");
  sand::SpecInfo info;
  const int rc = host_spec(spec, nullptr, nullptr, nullptr, &info);
  if (rc != SAND_OK) return rc;
  if (rank >= spec->world_size) return sand::set_error(SAND_EINVAL, "rank >= world_size");
  const std::vector<uint32_t> clips = sand::rank_clips(info, epoch, rank);
  if (clips.size() > cap) return sand::set_error(SAND_ERANGE, "output capacity too small");
  std::copy(clips.begin(), clips.end(), out);
  *n = static_cast<uint32_t>(clips.size());
  return SAND_OK;
}

extern "C" int sand_plan_clip(const sand_view_spec* spec, const uint32_t* n_frames, const uint32_t* widths,
                              const uint32_t* heights, uint64_t epoch, uint32_t clip, sand_clip_meta* out) {
  if (!out || !n_frames || !widths || !heights) return sand::set_error(SAND_EINVAL, "null argument");
  sand::SpecInfo info;
  const int rc = host_spec(spec, n_frames, widths, heights, &info);
  if (rc != SAND_OK) return rc;
  if (static_cast<uint64_t>(clip) >= static_cast<uint64_t>(spec->n_videos) * spec->samples_per_video)
    return sand::set_error(SAND_ERANGE, "clip id out of range");
  sand::plan_clip(info, epoch, clip, out);
  return SAND_OK;
}
