// mat_direct.cu — launcher of the direct-gather kernel for heavy down-scaling (k_direct.cuh).
#include <algorithm>

#include "kernels_common.cuh"
#include "k_direct.cuh"

namespace sand {

int launch_direct(const LaunchParams& p, const BatchShape& sh, cudaStream_t stream) {
  constexpr int RB = 32;
  const int pairs = (sh.heavy_max_wo + 1) / 2;
  const int P = std::min(112, pairs);                       // column pairs per CTA
  const int nchunks = (pairs + P - 1) / P;
  const int threads = ((2 * P + 31) / 32) * 32;             // two half-bands of P threads
  const int nbands = (sh.heavy_max_ho + RB - 1) / RB;
  const unsigned blocks = (unsigned)((uint64_t)p.n_items * nbands * nchunks);
  switch (sh.even_wo ? sh.dtype : -1) {
    case SAND_U8: k_direct<SAND_U8, true><<<blocks, threads, 0, stream>>>(p, RB, nbands, nchunks); break;
    case SAND_BF16: k_direct<SAND_BF16, true><<<blocks, threads, 0, stream>>>(p, RB, nbands, nchunks); break;
    case SAND_F32: k_direct<SAND_F32, true><<<blocks, threads, 0, stream>>>(p, RB, nbands, nchunks); break;
    default: k_direct<-1, false><<<blocks, threads, 0, stream>>>(p, RB, nbands, nchunks); break;
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_error(e, "k_direct launch");
  return SAND_OK;
}

}  // namespace sand
