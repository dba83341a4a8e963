// mat_plain.cu — launcher of the multi-frame plain kernel (k_plain.cuh).
#include "kernels_common.cuh"
#include "k_plain.cuh"
#include "k_plainw.cuh"

namespace sand {

#ifndef SAND_PLAIN_NP
#define SAND_PLAIN_NP 2       // column pairs per thread (k_plain.cuh)
#endif
constexpr int kNP = SAND_PLAIN_NP;
#ifndef SAND_PLAINW
#define SAND_PLAINW 1         // warp-granular k_plainw for widths <= 256 (k_plain otherwise)
#endif

int plain_cols_per_thread() { return 2 * kNP; }
#ifndef SAND_PW_FPC_THREADS
#define SAND_PW_FPC_THREADS 112   // k_plainw: two frames (four warps) per task at 224 columns
#endif
int plain_max_threads() { return SAND_PLAINW ? SAND_PW_FPC_THREADS : PlainBounds<kNP>::kThreads; }


#define SAND_PLAINW_KERNELS(X, NPJ)                                                                   \
  X(SAND_U8, 1, NPJ, false) X(SAND_U8, 2, NPJ, false) X(SAND_BF16, 1, NPJ, false) X(SAND_BF16, 2, NPJ, false) \
  X(SAND_F32, 1, NPJ, false) X(SAND_F32, 2, NPJ, false) X(SAND_BF16, 1, NPJ, true) X(SAND_BF16, 2, NPJ, true) \
  X(SAND_F32, 1, NPJ, true) X(SAND_F32, 2, NPJ, true)

static int configure_plainw() {
#define SAND_PW_ALLOW(DT, ND, NPJ, FOLD)                                                   \
  if (cudaError_t e = allow_smem(k_plainw<DT, ND, NPJ, FOLD>); e != cudaSuccess) \
    return cuda_error(e, "cudaFuncSetAttribute(k_plainw)");
  SAND_PLAINW_KERNELS(SAND_PW_ALLOW, 1)
  SAND_PLAINW_KERNELS(SAND_PW_ALLOW, 2)
#undef SAND_PW_ALLOW
  return SAND_OK;
}

#ifndef SAND_PW_PDL
#define SAND_PW_PDL 1
#endif
// launch with programmatic stream serialisation: consecutive batches' kernels on one stream overlap
// the next grid's prologue with this grid's tail (k_plainw waits on the previous grid before it
// touches frames or outputs)
template <typename K>
static void launch_pdl(K kernel, unsigned grid, unsigned threads, size_t smem, cudaStream_t stream,
                       const LaunchParams& p, const uint2* tasks, const pw::Shape& s) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(threads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = SAND_PW_PDL;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  (void)cudaLaunchKernelEx(&cfg, kernel, p, tasks, s);   // errors surface via cudaGetLastError
}

// k_plainw: one warp per frame of a task (k_plainw.cuh); *launched = false when the batch does
// not fit it (mixed dtypes, widths not a multiple of 4 or > 256, spans beyond kGWMax, items with
// more than two destinations)
static int launch_plainw(const LaunchParams& p, const BatchShape& sh, int fpc, cudaStream_t stream, bool* launched) {
  *launched = false;
  if (!SAND_PLAINW || sh.n_tasks_w == 0 || sh.dtype < 0 || !sh.wo_mod4 || sh.max_wo > 256 || sh.pl_gw_w > pw::kGWMax ||
      sh.pl_rb > pw::kMaxRB || fpc < 1 || sh.max_dests > 2)
    return SAND_OK;
  pw::Shape s;
  s.nsub = (fpc + pw::kFrames - 1) / pw::kFrames;
  s.gw = sh.pl_gw_w;
  const size_t smem = pw::smem_bytes(s);
  if (smem > 200 * 1024) return SAND_OK;
  const uint2* tasks = p.tasks + sh.task_first;
  const bool nd1 = sh.max_dests <= 1, fold = sh.fold != 0 && sh.dtype != SAND_U8;
  const bool narrow = sh.max_wo <= 128;
  const unsigned threads = 64u * pw::kFrames;
  const unsigned grid = sh.n_tasks_w * (unsigned)s.nsub;   // the k_plainw-eligible tasks (first)
#define SAND_PW_GO(NPJ)                                                                                     \
  do {                                                                                                       \
    switch (sh.dtype) {                                                                                      \
      case SAND_U8:                                                                                          \
        if (nd1) launch_pdl(k_plainw<SAND_U8, 1, NPJ, false>, grid, threads, smem, stream, p, tasks, s);       \
        else launch_pdl(k_plainw<SAND_U8, 2, NPJ, false>, grid, threads, smem, stream, p, tasks, s);           \
        break;                                                                                               \
      case SAND_BF16:                                                                                        \
        if (fold && nd1) launch_pdl(k_plainw<SAND_BF16, 1, NPJ, true>, grid, threads, smem, stream, p, tasks, s);  \
        else if (fold) launch_pdl(k_plainw<SAND_BF16, 2, NPJ, true>, grid, threads, smem, stream, p, tasks, s);    \
        else if (nd1) launch_pdl(k_plainw<SAND_BF16, 1, NPJ, false>, grid, threads, smem, stream, p, tasks, s);    \
        else launch_pdl(k_plainw<SAND_BF16, 2, NPJ, false>, grid, threads, smem, stream, p, tasks, s);             \
        break;                                                                                               \
      default:                                                                                               \
        if (fold && nd1) launch_pdl(k_plainw<SAND_F32, 1, NPJ, true>, grid, threads, smem, stream, p, tasks, s);   \
        else if (fold) launch_pdl(k_plainw<SAND_F32, 2, NPJ, true>, grid, threads, smem, stream, p, tasks, s);     \
        else if (nd1) launch_pdl(k_plainw<SAND_F32, 1, NPJ, false>, grid, threads, smem, stream, p, tasks, s);     \
        else launch_pdl(k_plainw<SAND_F32, 2, NPJ, false>, grid, threads, smem, stream, p, tasks, s);              \
        break;                                                                                               \
    }                                                                                                        \
  } while (0)
  if (narrow) SAND_PW_GO(1);
  else SAND_PW_GO(2);
#undef SAND_PW_GO
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_error(e, "k_plainw launch");
  *launched = true;
  return SAND_OK;
}

int configure_plain() {
  if (int rc = configure_plainw(); rc != SAND_OK) return rc;
  for (cudaError_t e : {allow_smem(k_plain<SAND_U8, 1, kNP, false>), allow_smem(k_plain<SAND_BF16, 1, kNP, false>),
                        allow_smem(k_plain<SAND_F32, 1, kNP, false>), allow_smem(k_plain<SAND_U8, 2, kNP, false>),
                        allow_smem(k_plain<SAND_BF16, 2, kNP, false>), allow_smem(k_plain<SAND_F32, 2, kNP, false>),
                        allow_smem(k_plain<SAND_BF16, 1, kNP, true>), allow_smem(k_plain<SAND_F32, 1, kNP, true>),
                        allow_smem(k_plain<SAND_BF16, 2, kNP, true>), allow_smem(k_plain<SAND_F32, 2, kNP, true>)})
    if (e != cudaSuccess) return cuda_error(e, "cudaFuncSetAttribute(k_plain)");
  return SAND_OK;
}

static int launch_plain_tasks(const LaunchParams& p, const BatchShape& sh, int fpc, int nq, cudaStream_t stream,
                              bool* launched);

int launch_plain(const LaunchParams& p, const BatchShape& sh_in, int fpc, int nq, cudaStream_t stream, bool* launched) {
  *launched = false;
  BatchShape sh = sh_in;
  if (int rc = launch_plainw(p, sh, fpc, stream, launched); rc != SAND_OK) return rc;
  if (*launched) {                      // k_plainw took the eligible tasks; k_plain the wider rest
    if (sh.n_tasks_w == sh.n_tasks) return SAND_OK;
    sh.task_first += sh.n_tasks_w;
    sh.n_tasks -= sh.n_tasks_w;
    *launched = false;   // if k_plain declines them too, the generic kernel redoes the whole class
    return launch_plain_tasks(p, sh, fpc, nq, stream, launched);
  }
  return launch_plain_tasks(p, sh, fpc, nq, stream, launched);
}

// k_plain over the tasks [task_first, task_first + n_tasks) of the batch
static int launch_plain_tasks(const LaunchParams& p, const BatchShape& sh, int fpc, int nq, cudaStream_t stream,
                              bool* launched) {
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
