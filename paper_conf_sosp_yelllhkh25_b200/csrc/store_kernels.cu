// store_kernels.cu — device side of sand_store_put_frame_batch (the HBM frame
// store): one CTA per frame copies its Y rows and interleaved-UV rows from a packed staging
// buffer into the frame's pitched slab slot. 16 B words when every row offset is 16-aligned,
// else 4 B words, else bytes. Pure data movement (no arithmetic of the method).
#include <cuda_runtime.h>
#include <stdint.h>

#include <string>

#include "internal.h"

namespace sand {

int set_error(int code, const std::string& msg);
int cuda_error(cudaError_t e, const char* what);

namespace {

template <typename T>
__global__ void __launch_bounds__(256) k_put_scatter(const uint8_t* __restrict__ src, uint64_t src_pitch,
                                                     uint64_t uv_offset, uint8_t* __restrict__ slab,
                                                     const PutDesc* __restrict__ desc) {
  const PutDesc d = desc[blockIdx.x];
  const uint32_t words = d.width / sizeof(T);          // per row (width % sizeof(T) == 0)
  const uint32_t rows = d.height + d.height / 2;       // Y rows then UV rows
  const uint8_t* fs = src + d.src;
  uint8_t* fd = slab + d.dst;
  for (uint32_t e = threadIdx.x; e < rows * words; e += blockDim.x) {
    const uint32_t r = e / words, w = e - r * words;
    const uint8_t* s = r < d.height ? fs + (uint64_t)r * src_pitch : fs + uv_offset + (uint64_t)(r - d.height) * src_pitch;
    reinterpret_cast<T*>(fd + (uint64_t)r * d.dst_pitch)[w] = __ldg(reinterpret_cast<const T*>(s) + w);
  }
}

}  // namespace

int launch_put_scatter(const uint8_t* src, uint64_t src_pitch, uint64_t uv_offset, uint8_t* slab,
                       const PutDesc* desc, uint32_t n, int word, cudaStream_t stream) {
  if (n == 0) return SAND_OK;
  if (word == 16) k_put_scatter<uint4><<<n, 256, 0, stream>>>(src, src_pitch, uv_offset, slab, desc);
  else if (word == 4) k_put_scatter<uint32_t><<<n, 256, 0, stream>>>(src, src_pitch, uv_offset, slab, desc);
  else k_put_scatter<uint8_t><<<n, 256, 0, stream>>>(src, src_pitch, uv_offset, slab, desc);
  const cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_error(e, "k_put_scatter launch");
  return SAND_OK;
}

}  // namespace sand
