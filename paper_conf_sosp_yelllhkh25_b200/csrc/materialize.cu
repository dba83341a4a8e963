// materialize.cu — per-batch dispatch of the materialisation kernels.
//
// A batch's work items arrive partitioned by class (view.cpp build_plan), each class with its
// own kernel, so one item's shape never changes the kernel of another:
//   [0, n_mild)            plain, source step <= 2  -> k_copy (identity scale) or k_plain
//                                                      (k_stream for mixed dtypes / odd widths)
//   [n_mild, n_direct)     plain, heavier down-scaling -> k_direct
//   [n_direct, n_items)    rotation and/or blur        -> k_stencil2 (k_stencil beyond smem)
// Batches with several classes run them on the caller's stream and a forked auxiliary stream
// (joined before return), so a class's grid tail is filled by the other's CTAs.
#include <cuda_runtime.h>

#include "internal.h"
#include "kernels.h"

namespace sand {

int configure_kernels(size_t stencil_smem) {
  (void)stencil_smem;
  int rc = configure_plain();
  if (rc == SAND_OK) rc = configure_stream();
  if (rc == SAND_OK) rc = configure_stencil();
  return rc;
}

int launch_materialize(const LaunchParams& p, const BatchShape& shape, size_t stencil_smem, int pl_fpc, int pl_nq,
                       cudaStream_t stream, cudaStream_t aux, cudaEvent_t fork, cudaEvent_t join, int* n_launched,
                       ClassEvents* ev) {
  auto mark = [&](int cls, bool end, cudaStream_t s) {
    if (!ev) return cudaSuccess;
    if (end) ev->used[cls] = true;
    return cudaEventRecord(end ? ev->end[cls] : ev->start[cls], s);
  };
  *n_launched = 0;
  if (p.n_items == 0) return SAND_OK;
  const uint32_t n_mild = shape.n_mild, n_heavy = shape.n_direct - shape.n_mild;
  const uint32_t n_stencil = p.n_items - shape.n_direct;
  const int classes = (n_mild > 0) + (n_heavy > 0) + (n_stencil > 0);
  const bool fork_ok = classes > 1 && aux && fork && join;
  cudaStream_t side = stream;
  if (fork_ok) {
    cudaError_t e = cudaEventRecord(fork, stream);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(aux, fork, 0);
    if (e != cudaSuccess) return cuda_error(e, "fork of the auxiliary stream");
    side = aux;
  }
  // the heaviest class first on the caller's stream, the others on the auxiliary stream
  if (n_stencil > 0) {
    LaunchParams ps = p;
    ps.items = p.items + shape.n_direct;
    ps.n_items = n_stencil;
    mark(2, false, stream);
    const int rc = launch_stencil(ps, shape, stencil_smem, stream);
    if (rc != SAND_OK) return rc;
    mark(2, true, stream);
    ++*n_launched;
  }
  if (n_heavy > 0) {
    LaunchParams ph = p;
    ph.items = p.items + n_mild;
    ph.n_items = n_heavy;
    cudaStream_t s = n_stencil > 0 ? side : stream;
    mark(1, false, s);
    const int rc = launch_direct(ph, shape, s);
    if (rc != SAND_OK) return rc;
    mark(1, true, s);
    ++*n_launched;
  }
  if (n_mild > 0) {
    LaunchParams pm = p;
    pm.n_items = n_mild;
    cudaStream_t s = (n_stencil > 0 || n_heavy > 0) ? side : stream;
    bool done = false;
    mark(0, false, s);
    int rc = launch_copy(pm, shape, s, &done);
    if (rc == SAND_OK && !done) rc = launch_plain(pm, shape, pl_fpc, pl_nq, s, &done);
    if (rc == SAND_OK && !done) rc = launch_stream_generic(pm, shape, s);
    if (rc != SAND_OK) return rc;
    mark(0, true, s);
    ++*n_launched;
  }
  if (fork_ok) {
    cudaError_t e = cudaEventRecord(join, aux);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(stream, join, 0);
    if (e != cudaSuccess) return cuda_error(e, "join of the auxiliary stream");
  }
  return SAND_OK;
}

}  // namespace sand
