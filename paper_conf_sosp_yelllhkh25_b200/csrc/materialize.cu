// materialize.cu — sm_100a kernels of the materialisation path.
//
//  * k_resample_{raw,gather} (k_resample.cuh): items without rotation/blur — banded resample,
//               one CTA per (work item, band of output rows).
//  * k_stencil: items with rotation and/or blur, one CTA per work item. Per channel: Q2 plane in shared
//               memory -> rotated Q3 plane -> separable blur in row strips (fp32
//               horizontal pass kept in shared memory) -> normalise -> store.
// Arithmetic follows DESIGN.md R#11-R#17 with explicit IEEE-rounded intrinsics
// (__fmul_rn / __fadd_rn / __fmaf_rn), so the result is bit-identical to the oracle.
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include <algorithm>
#include <cmath>
#include <map>
#include <mutex>
#include <tuple>
#include <cstdlib>
#include <string>

#include "plan_types.h"
#include "sand.h"

namespace sand {

int set_error(int code, const std::string& msg);
int cuda_error(cudaError_t e, const char* what);

namespace {

constexpr int kStripRows = 32;     // output rows per blur strip

// ---------------------------------------------------------------- a5: NV12 -> RGB (R#11)
__device__ __forceinline__ int clamp_u8(int v) { return min(max(v, 0), 255); }

__device__ __forceinline__ int nv12_chan(const uint8_t* __restrict__ Yp, const uint8_t* __restrict__ UVp,
                                         uint32_t pitch, int x, int y, int c) {
  const int Yv = __ldg(Yp + (size_t)y * pitch + x);
  const uint8_t* uvr = UVp + (size_t)(y >> 1) * pitch + (x & ~1);
  const int u = (int)__ldg(uvr) - 128;
  const int v = (int)__ldg(uvr + 1) - 128;
  const int yy = max(Yv - 16, 0) * 1220542 + (1 << 19);
  const int t = c == 0 ? 1673527 * v : (c == 1 ? -852492 * v - 409993 * u : 2116026 * u);
  return clamp_u8((yy + t) >> 20);
}

// ---------------------------------------------------------------- a6: bilinear (R#12)
__device__ __forceinline__ void src_tap(float sc, int off, int o, int lim, int org, int& i0, int& i1,
                                        float& lam) {
  float s = __fadd_rn(__fmul_rn(sc, __fadd_rn((float)(off + o), 0.5f)), -0.5f);
  s = fmaxf(s, 0.f);
  const int i = (int)s;
  lam = __fsub_rn(s, (float)i);
  i0 = org + i;
  i1 = org + min(i + 1, lim - 1);
}

__device__ __forceinline__ float lerp_rn(float lam, float a, float b) { return __fmaf_rn(lam, __fsub_rn(b, a), a); }

__device__ __forceinline__ int quant(float v) { return clamp_u8(__float2int_rn(v)); }

// ---------------------------------------------------------------- a10: normalise + store (R#17)
__device__ __forceinline__ void store_value(const LaunchParams& p, uint32_t dest, int c, int oy, int ox, int q) {
  const uint32_t k = dest >> 24, t = (dest >> 16) & 0xffu, b = dest & 0xffffu;
  const ViewConst& vc = p.views[k];
  const size_t plane = (size_t)vc.out_h * vc.out_w;
  const size_t idx = ((((size_t)b * 3 + c) * vc.T + t) * plane) + (size_t)oy * vc.out_w + ox;
  if (vc.dtype == SAND_U8) {
    static_cast<uint8_t*>(p.out[k])[idx] = (uint8_t)q;
  } else {
    const float y = __fmaf_rn((float)q, vc.a[c], vc.b[c]);
    if (vc.dtype == SAND_BF16)
      static_cast<__nv_bfloat16*>(p.out[k])[idx] = __float2bfloat16_rn(y);
    else
      static_cast<float*>(p.out[k])[idx] = y;
  }
}

// ---------------------------------------------------------------- k_stencil
__device__ __forceinline__ int reflect_idx(int i, int n) { return i < 0 ? -i : (i >= n ? 2 * (n - 1) - i : i); }

__global__ void __launch_bounds__(512) k_stencil(const LaunchParams p) {
  extern __shared__ __align__(16) uint8_t smem[];
  const WorkItem w = p.items[blockIdx.x];
  if (!(w.flags & 1u)) return;
  const GroupParams& g = p.groups[w.gp];
  const uint8_t* Yp = p.slab + w.y_off;
  const uint8_t* UVp = Yp + (size_t)w.pitch * w.src_h;
  const int Wo = g.out_w, Ho = g.out_h, n = Ho * Wo;
  uint8_t* q2 = smem;
  uint8_t* q3 = smem + ((n + 15) & ~15);
  float* strip = reinterpret_cast<float*>(smem + 2 * ((n + 15) & ~15));
  const float cx = (float)(Wo - 1) * 0.5f, cy = (float)(Ho - 1) * 0.5f;
  const float rc = g.rot_c, rs = g.rot_s, nrs = -g.rot_s;
  const int r = g.blur_r;

  for (int c = 0; c < 3; ++c) {
    // Q2: resample (+ flip) of channel c
    for (int pix = threadIdx.x; pix < n; pix += blockDim.x) {
      const int oy = pix / Wo, ox = pix - (pix / Wo) * Wo;
      const int oxm = g.flip ? Wo - 1 - ox : ox;
      int x0, x1, y0, y1;
      float lx, ly;
      src_tap(g.sc_x, g.off_x, oxm, g.lim_x, g.org_x, x0, x1, lx);
      src_tap(g.sc_y, g.off_y, oy, g.lim_y, g.org_y, y0, y1, ly);
      const float h0 = lerp_rn(lx, (float)nv12_chan(Yp, UVp, w.pitch, x0, y0, c),
                               (float)nv12_chan(Yp, UVp, w.pitch, x1, y0, c));
      const float h1 = lerp_rn(lx, (float)nv12_chan(Yp, UVp, w.pitch, x0, y1, c),
                               (float)nv12_chan(Yp, UVp, w.pitch, x1, y1, c));
      q2[pix] = (uint8_t)quant(lerp_rn(ly, h0, h1));
    }
    __syncthreads();
    const uint8_t* src = q2;
    if (g.rot_on) {   // a8: Q3 = rotate(Q2) about the centre, zero outside (R#15)
      for (int pix = threadIdx.x; pix < n; pix += blockDim.x) {
        const int oy = pix / Wo, ox = pix - (pix / Wo) * Wo;
        const float xc = __fsub_rn((float)ox, cx), yc = __fsub_rn((float)oy, cy);
        const float sx = __fadd_rn(__fadd_rn(__fmul_rn(rc, xc), __fmul_rn(nrs, yc)), cx);
        const float sy = __fadd_rn(__fadd_rn(__fmul_rn(rs, xc), __fmul_rn(rc, yc)), cy);
        const float fx = floorf(sx), fy = floorf(sy);
        const float lx = __fsub_rn(sx, fx), ly = __fsub_rn(sy, fy);
        const int x0 = (int)fx, y0 = (int)fy;
        float t[2][2];
#pragma unroll
        for (int dy = 0; dy < 2; ++dy)
#pragma unroll
          for (int dx = 0; dx < 2; ++dx) {
            const int xx = x0 + dx, yy = y0 + dy;
            t[dy][dx] = (xx >= 0 && xx < Wo && yy >= 0 && yy < Ho) ? (float)q2[yy * Wo + xx] : 0.f;
          }
        const float h0 = lerp_rn(lx, t[0][0], t[0][1]);
        const float h1 = lerp_rn(lx, t[1][0], t[1][1]);
        q3[pix] = (uint8_t)quant(lerp_rn(ly, h0, h1));
      }
      __syncthreads();
      src = q3;
    }
    if (g.blur_on) {  // a9: separable blur in strips of output rows (R#16)
      for (int ys = 0; ys < Ho; ys += kStripRows) {
        const int ye = min(ys + kStripRows, Ho);
        const int rows = ye - ys + 2 * r;       // strip row j <-> image row reflect(ys - r + j)
        for (int e = threadIdx.x; e < rows * Wo; e += blockDim.x) {
          const int j = e / Wo, x = e - (e / Wo) * Wo;
          const int yrow = reflect_idx(ys - r + j, Ho);
          float acc = 0.f;
          for (int i = 0; i <= 2 * r; ++i)
            acc = __fmaf_rn(g.blur_w[i], (float)src[yrow * Wo + reflect_idx(x + i - r, Wo)], acc);
          strip[j * Wo + x] = acc;
        }
        __syncthreads();
        for (int e = threadIdx.x; e < (ye - ys) * Wo; e += blockDim.x) {
          const int yl = e / Wo, x = e - (e / Wo) * Wo;
          float acc = 0.f;
          for (int i = 0; i <= 2 * r; ++i) acc = __fmaf_rn(g.blur_w[i], strip[(yl + i) * Wo + x], acc);
          const int q = quant(acc);
          for (uint32_t d = 0; d < w.n_dest; ++d) store_value(p, p.dests[w.dest_begin + d], c, ys + yl, x, q);
        }
        __syncthreads();
      }
    } else {
      for (int pix = threadIdx.x; pix < n; pix += blockDim.x) {
        const int oy = pix / Wo, ox = pix - (pix / Wo) * Wo;
        for (uint32_t d = 0; d < w.n_dest; ++d) store_value(p, p.dests[w.dest_begin + d], c, oy, ox, src[pix]);
      }
      __syncthreads();
    }
  }
}

}  // namespace
}  // namespace sand

#include "k_resample.cuh"
#include "k_stream.cuh"
#include "k_stencil.cuh"
#include "k_direct.cuh"
#include "k_copy.cuh"

namespace sand {

namespace {
// Shared-memory budget per resample CTA: 4 CTAs of 7 warps per SM (tunable for experiments).
size_t smem_budget() {
  static size_t b = [] {
    const char* e = getenv("SAND_SMEM_BUDGET_KB");
    return (size_t)(e ? atoi(e) : 55) * 1024;
  }();
  return b;
}

struct ResampleCfg {
  int mode;         // 0 gather, 1 raw bands, 2 stream, 3 direct
  int R;
  size_t smem;
  st::Shape st;
};

int env_int(const char* name, int dflt) {
  const char* e = getenv(name);
  return e ? atoi(e) : dflt;
}

// mode, band height and dynamic shared memory of the resample kernel for a batch shape
ResampleCfg choose_resample(const BatchShape& sh) {
  static const int kCands[] = {64, 48, 32, 24, 16, 12, 8, 4, 2, 1};
  const bool mild = sh.cols_bound <= 2 * sh.max_wo + 16 && sh.max_scy <= 2.0f;
  const size_t gwb = rs::a16((size_t)sh.cols_bound) + 16;
  static const int forced = env_int("SAND_RESAMPLE_MODE", -1);
  if (mild && sh.max_wo <= 512 && forced != 1 && forced != 0) {
    st::Shape s;
    s.S = env_int("SAND_STREAM_S", 8);
    s.SB = env_int("SAND_STREAM_SB", 32);
    s.nsb = (sh.max_ho + s.SB - 1) / s.SB;
    // rows one sub-band spans: y0 of its S output rows moves by <= ceil((S-1) * scy), plus
    // the first y0 and the last y1; the raw buffer holds a sub-band's new Y rows and their UV rows
    s.ring = (int)std::ceil((double)sh.max_scy * (s.S - 1)) + 2;
    s.raw_rows = s.ring + s.ring / 2 + 2;
    s.ring_magic = (uint32_t)((1ull << 32) / (uint64_t)s.ring + 1);
    s.opts = env_int("SAND_STREAM_OPTS", 0);
    s.gw = (int)gwb;
    ResampleCfg c{2, 0, st::smem_bytes(s, sh.max_wo), s};
    if (s.ring <= 255 && c.smem <= 200 * 1024) return c;
  }
  if (mild && forced != 0) {
    for (int r : kCands) {
      const size_t rows = (size_t)std::ceil((double)sh.max_scy * r) + 3;
      const size_t bytes = rs::tables_bytes(sh.max_wo, r) + rows * gwb + rs::a16((rows / 2 + 2) * gwb) + rows * gwb * 4;
      if (bytes <= smem_budget() || (r <= 8 && bytes <= 200 * 1024)) return {1, r, bytes, {}};
    }
  }
  if (forced != 0) return {3, env_int("SAND_DIRECT_RB", 32), 0, {}};   // heavy down-scaling: direct gather
  for (int r : kCands) {
    const int span = (int)std::ceil((double)sh.max_scy * r) + 3;
    const size_t rows = (size_t)std::min(2 * r, span);
    const size_t cols = (size_t)std::min(2 * sh.max_wo, sh.cols_bound);
    const size_t bytes = rs::tables_bytes(sh.max_wo, r) + rs::gather_meta_bytes(sh.max_wo, r) + rows * cols * 4;
    if ((bytes <= smem_budget() && span <= 32 * rs::kRowWords) || r == 1) return {0, r, bytes, {}};
  }
  return {0, 1, 0, {}};
}

// Grid of a persistent kernel: every resident CTA slot of the device (occupancy at this block
// size and shared memory), capped by the task count. Cached per (kernel, threads, smem).
template <typename K>
unsigned persistent_grid(K kernel, int threads, size_t smem, uint64_t tasks) {
  static std::mutex mu;
  static std::map<std::tuple<const void*, int, size_t>, unsigned> cache;
  const auto key = std::make_tuple(reinterpret_cast<const void*>(kernel), threads, smem);
  unsigned slots = 0;
  {
    std::lock_guard<std::mutex> lk(mu);
    auto it = cache.find(key);
    if (it != cache.end()) slots = it->second;
  }
  if (slots == 0) {
    int dev = 0, nsm = 0, nb = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&nb, kernel, threads, smem);
    const int cap = env_int("SAND_CTAS_PER_SM", 0);
    if (cap > 0) nb = std::min(nb, cap);
    slots = (unsigned)std::max(1, nsm) * (unsigned)std::max(1, nb);
    if (env_int("SAND_PERSIST", 1) == 0) slots = ~0u;   // one CTA per task (A/B switch)
    std::lock_guard<std::mutex> lk(mu);
    cache[key] = slots;
  }
  return (unsigned)std::min<uint64_t>(tasks, slots);
}

template <int DT, bool VEC>
int launch_resample_dt(const LaunchParams& p, const BatchShape& sh, cudaStream_t stream) {
  // identity-scale batches (every direct item samples the source 1:1): the lerps are dead
  // (lambda = 0), so the copy-convert kernel renders the same bits without them
  static const int copy_env = env_int("SAND_COPY", 1);
  if constexpr (VEC && DT >= 0) {
    if (copy_env && sh.direct_identity && sh.src_w_mod4 && sh.wo_mod4 && sh.max_wo <= 1024) {
      const int quads = sh.max_wo / 4;
      const int rpi = std::max(1, 256 / quads);
      const int threads = ((rpi * quads + 31) / 32) * 32;
      static const int RB = std::max(1, env_int("SAND_COPY_RB", 32));
      const int nbands = (sh.max_ho + RB - 1) / RB;
      k_copy<DT><<<(unsigned)((uint64_t)p.n_items * nbands), threads, 0, stream>>>(p, RB, nbands);
      cudaError_t e = cudaGetLastError();
      if (e != cudaSuccess) return cuda_error(e, "k_copy launch");
      return SAND_OK;
    }
  }
  const ResampleCfg cfg = choose_resample(sh);
  if (cfg.smem > 227 * 1024) return set_error(SAND_EINVAL, "resample tile exceeds shared memory (source crop too large)");
  const int pairs = (sh.max_wo + 1) / 2;
  if (cfg.mode == 2) {
    const uint64_t tasks = (uint64_t)p.n_items * cfg.st.nsb;
    static const int np_env = env_int("SAND_STREAM_NP", 2);
    if constexpr (VEC && DT >= 0) {
      if (sh.wo_mod4 && np_env == 2) {   // four columns per thread
        const int threads = (((pairs + 1) / 2 + 31) / 32) * 32;
        const unsigned blocks = persistent_grid(k_stream<DT, VEC, 2>, threads, cfg.smem, tasks);
        k_stream<DT, VEC, 2><<<blocks, threads, cfg.smem, stream>>>(p, cfg.st, sh.max_wo);
        cudaError_t e = cudaGetLastError();
        if (e != cudaSuccess) return cuda_error(e, "k_stream launch");
        return SAND_OK;
      }
    }
    const int threads = ((pairs + 31) / 32) * 32;
    const unsigned blocks = persistent_grid(k_stream<DT, VEC, 1>, threads, cfg.smem, tasks);
    k_stream<DT, VEC, 1><<<blocks, threads, cfg.smem, stream>>>(p, cfg.st, sh.max_wo);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_error(e, "k_stream launch");
    return SAND_OK;
  }
  const int nbands = (sh.max_ho + cfg.R - 1) / cfg.R;
  if (cfg.mode == 3) {
    const int P = std::min(112, pairs);                       // column pairs per CTA
    const int nchunks = (pairs + P - 1) / P;
    const int threads = ((2 * P + 31) / 32) * 32;             // two half-bands of P threads
    const unsigned blocks = (unsigned)((uint64_t)p.n_items * nbands * nchunks);
    k_direct<DT, VEC><<<blocks, threads, 0, stream>>>(p, cfg.R, nbands, nchunks);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_error(e, "k_direct launch");
    return SAND_OK;
  }
  const int threads = std::min(224, ((2 * pairs + 31) / 32) * 32);
  const unsigned blocks = (unsigned)((uint64_t)p.n_items * nbands);
  if (cfg.mode == 1)
    k_resample_raw<DT, VEC><<<blocks, threads, cfg.smem, stream>>>(p, cfg.R, nbands, sh.max_wo);
  else
    k_resample_gather<DT, VEC><<<blocks, threads, cfg.smem, stream>>>(p, cfg.R, nbands, sh.max_wo);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_error(e, "k_resample launch");
  return SAND_OK;
}

// stencil kernel shape: Q2 band height R such that 3 planes + band/Q3 region fit 227 KB
bool choose_stencil(const BatchShape& sh, sc::Shape* out, size_t* smem) {
  const size_t plane = rs::a16((size_t)sh.st_max_wo * sh.st_max_ho);
  const int gw = (int)rs::a16((size_t)sh.st_cols_bound) + 16;
  const bool mild = sh.st_cols_bound <= 2 * sh.st_max_wo + 16 && sh.st_max_scy <= 2.0f;
  if (!mild || sh.st_max_wo > 1024) return false;
  static const int kCands[] = {64, 48, 32, 24, 16, 12, 8, 4};
  for (int r : kCands) {
    const int rows = (int)std::ceil((double)sh.st_max_scy * r) + 3;
    const size_t band = sc::band_bytes(sh.st_max_wo, r, rows, gw);
    // the band/Q3 region takes everything the three planes leave (one CTA per SM anyway): a
    // larger rotation ring and taller blur strips
    const size_t rest = 3 * plane < (size_t)227 * 1024 ? (size_t)227 * 1024 - 3 * plane : 0;
    const size_t u = std::max(std::max(plane, band), rest);
    const size_t total = 3 * plane + u;
    if (total <= 227 * 1024) {
      *out = sc::Shape{r, gw, rows, plane, u, env_int("SAND_STENCIL_SKIP", 0)};
      *smem = total;
      return true;
    }
  }
  return false;
}

template <typename K>
cudaError_t allow_smem(K kernel) {
  cudaFuncAttributes fa;
  cudaError_t e = cudaFuncGetAttributes(&fa, kernel);
  if (e != cudaSuccess) return e;
  e = cudaFuncSetAttribute(kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024 - (int)fa.sharedSizeBytes);
  if (e != cudaSuccess) return e;
  return cudaFuncSetAttribute(kernel, cudaFuncAttributePreferredSharedMemoryCarveout, 100);
}
}  // namespace

size_t stencil_smem_bytes(int max_h, int max_w, int max_r) {
  const size_t n = ((size_t)max_h * max_w + 15) & ~(size_t)15;
  return 2 * n + (size_t)(kStripRows + 2 * max_r) * max_w * sizeof(float);
}

int configure_kernels(size_t stencil_smem) {
  {
    cudaError_t e = cudaSuccess;
    for (cudaError_t r : {allow_smem(k_resample_raw<-1, false>), allow_smem(k_resample_raw<SAND_U8, true>),
                          allow_smem(k_resample_raw<SAND_BF16, true>), allow_smem(k_resample_raw<SAND_F32, true>),
                          allow_smem(k_resample_gather<-1, false>), allow_smem(k_resample_gather<SAND_U8, true>),
                          allow_smem(k_resample_gather<SAND_BF16, true>), allow_smem(k_resample_gather<SAND_F32, true>),
                          allow_smem(k_stream<-1, false, 1>), allow_smem(k_stream<SAND_U8, true, 1>),
                          allow_smem(k_stream<SAND_BF16, true, 1>), allow_smem(k_stream<SAND_F32, true, 1>),
                          allow_smem(k_stream<SAND_U8, true, 2>), allow_smem(k_stream<SAND_BF16, true, 2>),
                          allow_smem(k_stream<SAND_F32, true, 2>),
                          allow_smem(k_stencil2<-1, false>), allow_smem(k_stencil2<SAND_U8, true>),
                          allow_smem(k_stencil2<SAND_BF16, true>), allow_smem(k_stencil2<SAND_F32, true>)})
      if (r != cudaSuccess) e = r;
    if (e != cudaSuccess) return cuda_error(e, "cudaFuncSetAttribute(k_resample)");
  }
  if (stencil_smem > 0) {
    if (stencil_smem > 227 * 1024) return set_error(SAND_EINVAL, "stencil shared memory exceeds 227 KB");
    cudaError_t e = cudaFuncSetAttribute(k_stencil, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)stencil_smem);
    if (e != cudaSuccess) return cuda_error(e, "cudaFuncSetAttribute(k_stencil)");
  }
  return SAND_OK;
}

int launch_materialize(const LaunchParams& p, const BatchShape& shape, size_t stencil_smem, cudaStream_t stream,
                       cudaStream_t aux, cudaEvent_t fork, cudaEvent_t join, int* n_launched) {
  *n_launched = 0;
  if (p.n_items == 0) return SAND_OK;
  // both kinds in one batch: the stencil kernel (one 227 KB CTA per SM) goes first on the
  // caller's stream, the direct kernel on the forked aux stream, whose CTAs take the SMs the
  // stencil grid's last wave leaves idle; the caller's stream joins the aux work
  const bool fork_direct = shape.has_direct && shape.has_stencil && aux && fork && join;
  cudaStream_t direct_stream = stream;
  if (fork_direct) {
    cudaError_t e = cudaEventRecord(fork, stream);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(aux, fork, 0);
    if (e != cudaSuccess) return cuda_error(e, "fork of the direct kernel");
    direct_stream = aux;
  }
  if (shape.has_stencil) {
    LaunchParams ps = p;
    ps.items = p.items + shape.n_direct;
    ps.n_items = p.n_items - shape.n_direct;
    sc::Shape scs;
    size_t smem2;
    if (getenv("SAND_STENCIL_V1") == nullptr && choose_stencil(shape, &scs, &smem2)) {
      const int dt = shape.even_wo ? shape.dtype : -1;
      if (dt == SAND_U8) k_stencil2<SAND_U8, true><<<ps.n_items, 512, smem2, stream>>>(ps, scs, shape.st_max_wo);
      else if (dt == SAND_BF16) k_stencil2<SAND_BF16, true><<<ps.n_items, 512, smem2, stream>>>(ps, scs, shape.st_max_wo);
      else if (dt == SAND_F32) k_stencil2<SAND_F32, true><<<ps.n_items, 512, smem2, stream>>>(ps, scs, shape.st_max_wo);
      else k_stencil2<-1, false><<<ps.n_items, 512, smem2, stream>>>(ps, scs, shape.st_max_wo);
      cudaError_t e = cudaGetLastError();
      if (e != cudaSuccess) return cuda_error(e, "k_stencil2 launch");
    } else {
      k_stencil<<<ps.n_items, 512, stencil_smem, stream>>>(ps);
      cudaError_t e = cudaGetLastError();
      if (e != cudaSuccess) return cuda_error(e, "k_stencil launch");
    }
    ++*n_launched;
  }
  if (shape.has_direct) {
    LaunchParams pd = p;
    pd.n_items = shape.n_direct;
    int rc;
    // specialised instantiations: one dtype for every view and even output widths (the
    // 4-byte pair stores are aligned); anything else takes the generic instantiation
    switch (shape.even_wo ? shape.dtype : -1) {
      case SAND_U8: rc = launch_resample_dt<SAND_U8, true>(pd, shape, direct_stream); break;
      case SAND_BF16: rc = launch_resample_dt<SAND_BF16, true>(pd, shape, direct_stream); break;
      case SAND_F32: rc = launch_resample_dt<SAND_F32, true>(pd, shape, direct_stream); break;
      default: rc = launch_resample_dt<-1, false>(pd, shape, direct_stream); break;
    }
    if (rc != SAND_OK) return rc;
    ++*n_launched;
  }
  if (fork_direct) {
    cudaError_t e = cudaEventRecord(join, aux);
    if (e == cudaSuccess) e = cudaStreamWaitEvent(stream, join, 0);
    if (e != cudaSuccess) return cuda_error(e, "join of the direct kernel");
  }
  return SAND_OK;
}

}  // namespace sand
