// mat_crop.cu — launcher of the cached-object crop kernel (k_crop.cuh).
#include "kernels_common.cuh"
#include "k_crop.cuh"

namespace sand {

int launch_crop(const LaunchParams& p, const uint8_t* slab, const void* items, uint32_t n_items, int max_wo,
                int max_ho, int dtype, cudaStream_t stream) {
  if (n_items == 0) return SAND_OK;
  if (max_wo % 4) return set_error(SAND_EINVAL, "cached crops need out_w % 4 == 0");
  const int quads = max_wo / 4;
  const int rpi = quads >= 256 ? 1 : 256 / quads;
  const int threads = ((rpi * quads + 31) / 32) * 32;
  const int nbands = (max_ho + kCropRB - 1) / kCropRB;
  const unsigned blocks = n_items * (unsigned)nbands;
  const auto* it = static_cast<const CropItem*>(items);
  switch (dtype) {
    case SAND_U8: k_crop<SAND_U8><<<blocks, threads, 0, stream>>>(p, slab, it, nbands); break;
    case SAND_BF16: k_crop<SAND_BF16><<<blocks, threads, 0, stream>>>(p, slab, it, nbands); break;
    default: k_crop<SAND_F32><<<blocks, threads, 0, stream>>>(p, slab, it, nbands); break;
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_error(e, "k_crop launch");
  return SAND_OK;
}

}  // namespace sand
