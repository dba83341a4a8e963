// sand_api.cpp — error reporting and version of the C-ABI (include/sand.h).
#include <cuda_runtime.h>

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
