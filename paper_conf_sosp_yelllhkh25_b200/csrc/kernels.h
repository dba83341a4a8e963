// kernels.h — host-side interface of the kernel translation units (mat_*.cu) to the dispatcher
// (materialize.cu). Each launcher enqueues one kernel on `stream` and returns SAND_OK or a
// SAND_E* code (message via set_error); none synchronises.
#pragma once
#include <cuda_runtime.h>
#include <stddef.h>
#include <stdint.h>

#include <string>

#include "plan_types.h"
#include "sand.h"

namespace sand {

int set_error(int code, const std::string& msg);
int cuda_error(cudaError_t e, const char* what);

// Opt every kernel of a unit into the full 227 KB of dynamic shared memory (minus its static
// shared memory) on the current device; called once per view (view.cpp).
int configure_plain();
int configure_stream();
int configure_stencil();

// mat_plain.cu — k_plain over mild items p.items[0, n) using the batch's task slice. Returns
// SAND_OK with *launched = false when the batch does not fit k_plain (mixed dtypes, widths not a
// multiple of 4, shared memory); the caller then takes the generic kernel.
int launch_plain(const LaunchParams& p, const BatchShape& sh, int fpc, int nq, cudaStream_t stream, bool* launched);
// k_plain's output columns per thread and largest CTA (the view sizes its tasks from them)
int plain_cols_per_thread();
int plain_max_threads();

// mat_stream.cu — identity-scale copy kernel (k_copy; *launched = false if not applicable) and
// the generic streaming kernel (k_stream, any dtype mix / width) over mild items p.items[0, n)
int launch_copy(const LaunchParams& p, const BatchShape& sh, cudaStream_t stream, bool* launched);
int launch_stream_generic(const LaunchParams& p, const BatchShape& sh, cudaStream_t stream);

// mat_direct.cu — k_direct over heavy items p.items[0, n) (source step > 2)
int launch_direct(const LaunchParams& p, const BatchShape& sh, cudaStream_t stream);

// mat_crop.cu — crops of cached resized frames (f2): `items` is a device array of n_items
// CropItem (k_crop.cuh), all of one output dtype
int launch_crop(const LaunchParams& p, const uint8_t* slab, const void* items, uint32_t n_items, int max_wo,
                int max_ho, int dtype, cudaStream_t stream);

// mat_stencil.cu — rotation / blur items p.items[0, n): k_stencil2, or k_stencil for planes
// beyond shared memory
size_t stencil_smem_bytes(int max_h, int max_w, int max_r);
int launch_stencil(const LaunchParams& p, const BatchShape& sh, size_t stencil_smem, cudaStream_t stream);

// allow the full dynamic shared memory of one kernel (shared by the units)
template <typename K>
cudaError_t allow_smem(K kernel) {
  cudaFuncAttributes fa;
  cudaError_t e = cudaFuncGetAttributes(&fa, kernel);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024 - (int)fa.sharedSizeBytes);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(kernel, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
}

}  // namespace sand
