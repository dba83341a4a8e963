// mat_stream.cu — launchers of the identity-scale copy kernel (k_copy.cuh) and the generic
// streaming kernel (k_stream.cuh, any dtype mix and width; the fallback of k_plain).
#include <algorithm>
#include <cmath>
#include <map>
#include <mutex>
#include <tuple>

#include "kernels_common.cuh"
#include "k_copy.cuh"

namespace sand {

int configure_stream() {
  cudaError_t e = allow_smem(k_stream<-1, false, 1>);
  if (e != cudaSuccess) return cuda_error(e, "cudaFuncSetAttribute(k_stream)");
  return SAND_OK;
}

int launch_copy(const LaunchParams& p, const BatchShape& sh, cudaStream_t stream, bool* launched) {
  *launched = false;
  // every mild item samples its source 1:1 (lambda = 0 everywhere, R#12): the lerps are dead
  // and the copy-convert kernel renders the same bits without them
  if (!(sh.direct_identity && sh.src_w_mod4 && sh.wo_mod4 && sh.dtype >= 0 && sh.max_wo <= 1024)) return SAND_OK;
  const int quads = sh.max_wo / 4;
  const int rpi = std::max(1, 256 / quads);
  const int threads = ((rpi * quads + 31) / 32) * 32;
  constexpr int RB = 32;
  const int nbands = (sh.max_ho + RB - 1) / RB;
  const unsigned blocks = (unsigned)((uint64_t)p.n_items * nbands);
  const bool fold = sh.fold != 0;   // normalisation folds the rint bias (ViewConst::fold)
  switch (sh.dtype) {
    case SAND_U8: k_copy<SAND_U8, false><<<blocks, threads, 0, stream>>>(p, RB, nbands); break;
    case SAND_BF16:
      if (fold) k_copy<SAND_BF16, true><<<blocks, threads, 0, stream>>>(p, RB, nbands);
      else k_copy<SAND_BF16, false><<<blocks, threads, 0, stream>>>(p, RB, nbands);
      break;
    default:
      if (fold) k_copy<SAND_F32, true><<<blocks, threads, 0, stream>>>(p, RB, nbands);
      else k_copy<SAND_F32, false><<<blocks, threads, 0, stream>>>(p, RB, nbands);
      break;
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_error(e, "k_copy launch");
  *launched = true;
  return SAND_OK;
}

int launch_stream_generic(const LaunchParams& p, const BatchShape& sh, cudaStream_t stream) {
  st::Shape s;
  s.S = 8;
  s.SB = 32;
  s.nsb = (sh.max_ho + s.SB - 1) / s.SB;
  // rows one sub-band spans: y0 of its S output rows moves by <= ceil((S - 1) * scy), plus the
  // first y0 and the last y1; the staging buffer holds a sub-band's new Y rows and their UV rows
  s.ring = (int)std::ceil((double)sh.max_scy * (s.S - 1)) + 2;
  s.raw_rows = s.ring + s.ring / 2 + 2;
  s.ring_magic = (uint32_t)((1ull << 32) / (uint64_t)s.ring + 1);
  s.opts = 0;
  s.gw = (int)rs::a16((size_t)sh.cols_bound) + 16;   // >= every item's exact 16-aligned span
  const size_t smem = st::smem_bytes(s, sh.max_wo);
  if (smem > 200 * 1024 || s.ring > 255)
    return set_error(SAND_EINVAL, "resample tile exceeds shared memory (output too wide for the generic kernel)");
  const int pairs = (sh.max_wo + 1) / 2;
  const int threads = ((pairs + 31) / 32) * 32;
  // persistent CTAs: every resident slot of the device, capped by the task count
  static std::mutex mu;
  static std::map<std::tuple<int, int, size_t>, unsigned> cache;
  int dev = 0;
  cudaGetDevice(&dev);
  unsigned slots;
  {
    std::lock_guard<std::mutex> lk(mu);
    auto key = std::make_tuple(dev, threads, smem);
    auto it = cache.find(key);
    if (it == cache.end()) {
      int nsm = 0, nb = 0;
      cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
      cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, k_stream<-1, false, 1>, threads, smem);
      it = cache.emplace(key, (unsigned)std::max(1, nsm) * (unsigned)std::max(1, nb)).first;
    }
    slots = it->second;
  }
  const uint64_t tasks = (uint64_t)p.n_items * s.nsb;
  const unsigned blocks = (unsigned)std::min<uint64_t>(tasks, slots);
  k_stream<-1, false, 1><<<blocks, threads, smem, stream>>>(p, s, sh.max_wo);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_error(e, "k_stream launch");
  return SAND_OK;
}

}  // namespace sand
