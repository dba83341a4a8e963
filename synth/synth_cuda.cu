/*
 * synth_cuda.cu — device side of the synthetic NV12 generator (see nv12_synth.h).
 * Built into libsynth_cuda.so; bench.py and the GPU tests use it to fill large
 * frame stores directly in HBM (a 40 GB store cannot be generated on the host).
 * Bit-identical to synth.c because both evaluate the same pure byte function.
 */
#include <cuda_runtime.h>
#include <stdint.h>
#include "nv12_synth.h"

/* one thread per 4-byte word of one row of one plane of one frame */
__global__ void synth_fill_kernel(int family, uint64_t seed, uint32_t video, uint32_t first_frame,
                                  uint32_t width, uint32_t height, uint8_t* y, size_t y_pitch,
                                  uint8_t* uv, size_t uv_pitch, size_t frame_stride) {
  const uint32_t f = blockIdx.z;
  const uint32_t row_all = blockIdx.y;            /* 0..H-1 Y rows, then H/2 UV rows */
  const uint32_t plane = row_all < height ? 0u : 1u;
  const uint32_t r = plane == 0 ? row_all : row_all - height;
  const uint32_t frame = first_frame + f;
  uint8_t* row = (plane == 0 ? y + (size_t)r * y_pitch : uv + (size_t)r * uv_pitch) + (size_t)f * frame_stride;
  const uint32_t key = synth_row_key(seed, video, frame, plane, r);
  for (uint32_t q = blockIdx.x * blockDim.x + threadIdx.x; q * 4u < width; q += gridDim.x * blockDim.x) {
    uint32_t c = q * 4u;
    uint32_t w;
    if (family == SYNTH_SMOOTH) {
      w = 0;
      for (uint32_t k = 0; k < 4; ++k)
        if (c + k < width) w |= (uint32_t)synth_smooth_byte(seed, video, frame, plane, r, c + k) << (8 * k);
    } else {
      w = synth_uniform_word(key, q);
    }
    if (c + 4 <= width && ((((uintptr_t)(row + c)) & 3u) == 0)) {
      *reinterpret_cast<uint32_t*>(row + c) = w;
    } else {
      for (uint32_t k = 0; k < 4 && c + k < width; ++k) row[c + k] = (uint8_t)(w >> (8 * k));
    }
  }
}

extern "C" int synth_fill_frames_cuda(int family, uint64_t seed, uint32_t video, uint32_t first_frame,
                                      uint32_t n_frames, uint32_t width, uint32_t height,
                                      uint8_t* y, size_t y_pitch, uint8_t* uv, size_t uv_pitch,
                                      size_t frame_stride, cudaStream_t stream) {
  if ((width & 1u) || (height & 1u) || width == 0 || height == 0 || n_frames == 0) return -1;
  if (n_frames > 65535u) return -1;
  dim3 block(128);
  uint32_t words = (width + 3u) / 4u;
  dim3 grid((words + block.x - 1) / block.x, height + height / 2, n_frames);
  synth_fill_kernel<<<grid, block, 0, stream>>>(family, seed, video, first_frame, width, height, y,
                                                y_pitch, uv, uv_pitch, frame_stride);
  return cudaGetLastError() == cudaSuccess ? 0 : -5;
}
