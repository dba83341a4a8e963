// mat_plain.cu — launcher of the multi-frame plain kernel (k_plain.cuh).
#include "kernels_common.cuh"
#include "k_plain.cuh"

namespace sand {

int configure_plain() {
  for (cudaError_t e : {allow_smem(k_plain<SAND_U8, 1>), allow_smem(k_plain<SAND_BF16, 1>),
                        allow_smem(k_plain<SAND_F32, 1>), allow_smem(k_plain<SAND_U8, 2>),
                        allow_smem(k_plain<SAND_BF16, 2>), allow_smem(k_plain<SAND_F32, 2>)})
    if (e != cudaSuccess) return cuda_error(e, "cudaFuncSetAttribute(k_plain)");
  return SAND_OK;
}

int launch_plain(const LaunchParams& p, const BatchShape& sh, int fpc, int nq, cudaStream_t stream, bool* launched) {
  *launched = false;
  if (sh.n_tasks == 0 || !sh.wo_mod4 || sh.dtype < 0) return SAND_OK;
  pl::Shape s;
  s.fpc = fpc;
  s.nq = nq;
  s.S = kPlainS;
  s.rb = sh.pl_rb;
  s.ring = sh.pl_ring;
  s.raw_rows = sh.pl_raw;
  s.gw = sh.pl_gw;
  s.ring_magic = (uint32_t)((1ull << 32) / (uint64_t)s.ring + 1);
  const size_t smem = pl::smem_bytes(s);
  if (smem > 200 * 1024 || s.ring > 255) return SAND_OK;       // pathological shapes: generic kernel
  const unsigned threads = (unsigned)((fpc * nq + 31) / 32 * 32);
  if (threads > 224) return SAND_OK;                             // outputs wider than 896: generic kernel
  const uint2* tasks = p.tasks + sh.task_first;
  const bool nd1 = sh.max_dests <= 1;
  switch (sh.dtype) {
    case SAND_U8:
      if (nd1) k_plain<SAND_U8, 1><<<sh.n_tasks, threads, smem, stream>>>(p, tasks, s);
      else k_plain<SAND_U8, 2><<<sh.n_tasks, threads, smem, stream>>>(p, tasks, s);
      break;
    case SAND_BF16:
      if (nd1) k_plain<SAND_BF16, 1><<<sh.n_tasks, threads, smem, stream>>>(p, tasks, s);
      else k_plain<SAND_BF16, 2><<<sh.n_tasks, threads, smem, stream>>>(p, tasks, s);
      break;
    default:
      if (nd1) k_plain<SAND_F32, 1><<<sh.n_tasks, threads, smem, stream>>>(p, tasks, s);
      else k_plain<SAND_F32, 2><<<sh.n_tasks, threads, smem, stream>>>(p, tasks, s);
      break;
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_error(e, "k_plain launch");
  *launched = true;
  return SAND_OK;
}

}  // namespace sand
