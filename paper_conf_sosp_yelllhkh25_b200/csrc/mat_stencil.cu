// mat_stencil.cu — items with rotation and/or blur (two-view config):
// launcher of k_stencil2 (k_stencil.cuh), and k_stencil, the per-channel fallback for output
// planes beyond shared memory. Per channel: Q2 plane in shared memory -> rotated Q3 plane ->
// separable blur in row strips (fp32 horizontal pass kept in shared memory) -> normalise ->
// store. Arithmetic follows DESIGN.md R#11-R#17 with explicit IEEE-rounded intrinsics
// (__fmul_rn / __fadd_rn / __fmaf_rn), so the result is bit-identical to the oracle.
#include <algorithm>
#include <cmath>

#include "kernels_common.cuh"
#include "k_stencil.cuh"

namespace sand {

namespace {

constexpr int kStripRows = 32;     // output rows per blur strip

// ---------------------------------------------------------------- a5: NV12 -> RGB (R#11)
__device__ __forceinline__ int clamp_u8(int v) { return min(max(v, 0), 255); }

__device__ __forceinline__ int nv12_chan(const uint8_t* __restrict__ Yp, const uint8_t* __restrict__ UVp,
                                         uint32_t pitch, int x, int y, int c, const ColorM& m) {
  const int Yv = __ldg(Yp + (size_t)y * pitch + x);
  const uint8_t* uvr = UVp + (size_t)(y >> 1) * pitch + (x & ~1);
  const int u = (int)__ldg(uvr) - 128;
  const int v = (int)__ldg(uvr + 1) - 128;
  const int yy = max(Yv - 16, 0) * m.cy + (1 << 19);
  const int t = c == 0 ? m.vr * v : (c == 1 ? m.vg * v + m.ug * u : m.ub * u);
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
      const float h0 = lerp_rn(lx, (float)nv12_chan(Yp, UVp, w.pitch, x0, y0, c, p.cm),
                               (float)nv12_chan(Yp, UVp, w.pitch, x1, y0, c, p.cm));
      const float h1 = lerp_rn(lx, (float)nv12_chan(Yp, UVp, w.pitch, x0, y1, c, p.cm),
                               (float)nv12_chan(Yp, UVp, w.pitch, x1, y1, c, p.cm));
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

namespace {
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
      *out = sc::Shape{r, gw, rows, plane, u};
      *smem = total;
      return true;
    }
  }
  return false;
}

}  // namespace

int configure_stencil() {
  for (cudaError_t e : {allow_smem(k_stencil2<-1, false>), allow_smem(k_stencil2<SAND_U8, true>),
                        allow_smem(k_stencil2<SAND_BF16, true>), allow_smem(k_stencil2<SAND_F32, true>),
                        allow_smem(k_stencil)})
    if (e != cudaSuccess) return cuda_error(e, "cudaFuncSetAttribute(k_stencil)");
  return SAND_OK;
}

size_t stencil_smem_bytes(int max_h, int max_w, int max_r) {
  const size_t n = ((size_t)max_h * max_w + 15) & ~(size_t)15;
  return 2 * n + (size_t)(kStripRows + 2 * max_r) * max_w * sizeof(float);
}

int launch_stencil(const LaunchParams& ps, const BatchShape& shape, size_t stencil_smem, cudaStream_t stream) {
  sc::Shape scs;
  size_t smem2;
  if (choose_stencil(shape, &scs, &smem2)) {
    const int dt = shape.even_wo ? shape.dtype : -1;
    if (dt == SAND_U8) k_stencil2<SAND_U8, true><<<ps.n_items, 512, smem2, stream>>>(ps, scs, shape.st_max_wo);
    else if (dt == SAND_BF16) k_stencil2<SAND_BF16, true><<<ps.n_items, 512, smem2, stream>>>(ps, scs, shape.st_max_wo);
    else if (dt == SAND_F32) k_stencil2<SAND_F32, true><<<ps.n_items, 512, smem2, stream>>>(ps, scs, shape.st_max_wo);
    else k_stencil2<-1, false><<<ps.n_items, 512, smem2, stream>>>(ps, scs, shape.st_max_wo);
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return cuda_error(e, "k_stencil2 launch");
    return SAND_OK;
  }
  if (stencil_smem > 227 * 1024) return set_error(SAND_EINVAL, "stencil planes exceed shared memory");
  if (shape.has_jitter)   // the per-channel fallback has no 3-plane stage for the jitter (R#30)
    return set_error(SAND_EINVAL, "colour jitter needs crops with a source step <= 2 (k_stencil2)");
  k_stencil<<<ps.n_items, 512, stencil_smem, stream>>>(ps);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return cuda_error(e, "k_stencil launch");
  return SAND_OK;
}

}  // namespace sand
