// mat_plain.cu — launcher of the multi-frame plain kernel (k_plain.cuh).
#include "kernels_common.cuh"
#include "k_plain.cuh"

namespace sand {

#ifndef SAND_PLAIN_NP
#define SAND_PLAIN_NP 2       // column pairs per thread (k_plain.cuh)
#endif
constexpr int kNP = SAND_PLAIN_NP;

int plain_cols_per_thread() { return 2 * kNP; }
int plain_max_threads() { return PlainBounds<kNP>::kThreads; }

int configure_plain() {
  for (cudaError_t e : {allow_smem(k_plain<SAND_U8, 1, kNP, false>), allow_smem(k_plain<SAND_BF16, 1, kNP, false>),
                        allow_smem(k_plain<SAND_F32, 1, kNP, false>), allow_smem(k_plain<SAND_U8, 2, kNP, false>),
                        allow_smem(k_plain<SAND_BF16, 2, kNP, false>), allow_smem(k_plain<SAND_F32, 2, kNP, false>),
                        allow_smem(k_plain<SAND_BF16, 1, kNP, true>), allow_smem(k_plain<SAND_F32, 1, kNP, true>),
                        allow_smem(k_plain<SAND_BF16, 2, kNP, true>), allow_smem(k_plain<SAND_F32, 2, kNP, true>)})
    if (e != cudaSuccess) return cuda_error(e, "cudaFuncSetAttribute(k_plain)");
  return SAND_OK;
}

int launch_plain(const LaunchParams& p, const BatchShape& sh, int fpc, int nq, cudaStream_t stream, bool* launched) {
  *launched = false;
  if (sh.n_tasks == 0 || sh.dtype < 0 || (kNP == 2 ? !sh.wo_mod4 : !sh.even_wo)) return SAND_OK;
  pl::Shape s;
  s.fpc = fpc;
  s.nq = nq;
  s.rb = sh.pl_rb;
  s.gw = sh.pl_gw;
  const size_t smem = pl::smem_bytes(s);
  if (smem > 200 * 1024) return SAND_OK;                         // pathological widths: generic kernel
  const unsigned threads = (unsigned)((fpc * nq + 31) / 32 * 32);
  if (threads > (unsigned)PlainBounds<kNP>::kThreads) return SAND_OK;   // very wide outputs: generic kernel
  if (sh.max_wo > 2 * kNP * nq) return SAND_OK;                   // wider than the view's CTA rows
  const uint2* tasks = p.tasks + sh.task_first;
  const bool nd1 = sh.max_dests <= 1;
#define SAND_PLAIN_LAUNCH(DT, ND, FOLD) k_plain<DT, ND, kNP, FOLD><<<sh.n_tasks, threads, smem, stream>>>(p, tasks, s)
  const bool fold = sh.fold != 0;   // normalisation folds the rint bias (ViewConst::fold)
  switch (sh.dtype) {
    case SAND_U8:
      if (nd1) SAND_PLAIN_LAUNCH(SAND_U8, 1, false);
      else SAND_PLAIN_LAUNCH(SAND_U8, 2, false);
      break;
    case SAND_BF16:
      if (fold) {
        if (nd1) SAND_PLAIN_LAUNCH(SAND_BF16, 1, true);
        else SAND_PLAIN_LAUNCH(SAND_BF16, 2, true);
      } else {
        if (nd1) SAND_PLAIN_LAUNCH(SAND_BF16, 1, false);
        else SAND_PLAIN_LAUNCH(SAND_BF16, 2, false);
      }
      break;
    default:
      if (fold) {
        if (nd1) SAND_PLAIN_LAUNCH(SAND_F32, 1, true);
        else SAND_PLAIN_LAUNCH(SAND_F32, 2, true);
      } else {
        if (nd1) SAND_PLAIN_LAUNCH(SAND_F32, 1, false);
        else SAND_PLAIN_LAUNCH(SAND_F32, 2, false);
      }
      break;
  }
#undef SAND_PLAIN_LAUNCH
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_error(e, "k_plain launch");
  *launched = true;
  return SAND_OK;
}

}  // namespace sand
