// k_resample.cuh — fused resample kernel for items without rotation/blur
// (DESIGN.md §7).
//
// One CTA = one work item (clip slot, source frame, group) x one band of R output rows.
//  1. Separable tap tables: output column j -> (x0, x1, lambda_x); band row -> (y0, y1,
//     lambda_y) with the exact fp32 rule of R#12.
//  2. Source -> shared memory, two modes chosen per batch by the host:
//     RAW    (scale <= ~2, Kinetics/SlowFast): the band's NV12 footprint (Y rows + UV rows,
//            16 B aligned column span) is copied with cp.async (LDGSTS, all requests in
//            flight at once), then converted in shared memory to packed RGBx, two pixels
//            per thread sharing one chroma sample (a4, a5, Q1).
//     GATHER (heavy down-scaling, 1080p Ray trials): only the tapped source columns and
//            rows are touched: bitmaps + popcount prefix give a compact tap grid, whose
//            pixels are gathered from HBM with 4 independent loads in flight per thread
//            and converted (a4, a5).
//  3. Two row-walker groups; each thread owns two adjacent output columns, walks down its
//     half of the band and keeps the horizontal lerps of the two current source rows in
//     registers, so each (source row, column) lerp is computed once (a6). Flip is the
//     column mirror (a7). Vertical lerp, rint, normalise and packing run as FFMA2/FADD2
//     pairs (sm_100a packed fp32), then one 4-byte store per (row, channel, destination)
//     through per-destination pointers computed once (a10); every destination view of the
//     group is written from the same registers (a11, node merging P:L277).
// Every fp32 operation is the R#12/R#17 op sequence with IEEE rounding, so results are
// bit-identical to the oracle (byte->float via the 2^23 exponent trick and rint via
// +1.5*2^23 are exact for values in [0, 256)).
#pragma once

namespace sand {
namespace rs {

constexpr int kColWords = 128;             // GATHER: source column span <= 4096
constexpr int kRowWords = 32;              // GATHER: band source row span <= 1024
constexpr int kInlineDests = 2;            // destinations kept in registers
constexpr float kBias = 8388608.0f;        // 2^23
constexpr float kRound = 12582912.0f;      // 1.5 * 2^23

__host__ __device__ inline size_t a16(size_t x) { return (x + 15) & ~size_t(15); }

// --- shared layout: [tables][mode data] -----------------------------------------------
struct Tables {
  uint2* ctab;        // per output column j: (x0 | x1 << 16 grid-relative, bits of lambda_x)
  uint2* rtab;        // per band row: (y0 | y1 << 16 grid-relative, bits of lambda_y)
  int* misc;          // GATHER: [0] tapped columns, [1] tapped rows
};

__host__ __device__ inline size_t tables_bytes(int maxWo, int R) {
  return a16((size_t)maxWo * 8) + a16((size_t)R * 8) + 16;
}

__device__ inline Tables carve_tables(uint8_t*& p, int maxWo, int R) {
  Tables t;
  t.ctab = reinterpret_cast<uint2*>(p); p += a16((size_t)maxWo * 8);
  t.rtab = reinterpret_cast<uint2*>(p); p += a16((size_t)R * 8);
  t.misc = reinterpret_cast<int*>(p); p += 16;
  return t;
}

// GATHER-mode bookkeeping
__host__ __device__ inline size_t gather_meta_bytes(int maxWo, int R) {
  return a16(kColWords * 4) + a16(kRowWords * 4) + a16(kColWords * 2) + a16(kRowWords * 2) +
         a16((size_t)2 * maxWo * 2) + a16((size_t)2 * R * 2);
}

// source tap of output index o (R#12): s = max(sc*((float)(off+o)+0.5f)-0.5f, 0)
__device__ __forceinline__ void tap(float sc, int off, int o, int lim, int org, int& i0, int& i1, float& lam) {
  float s = __fadd_rn(__fmul_rn(sc, __fadd_rn((float)(off + o), 0.5f)), -0.5f);
  s = fmaxf(s, 0.f);
  const int i = (int)s;
  lam = __fsub_rn(s, (float)i);
  i0 = org + i;
  i1 = org + min(i + 1, lim - 1);
}

__device__ __forceinline__ int tap0(float sc, int off, int o, int org) {
  float s = __fadd_rn(__fmul_rn(sc, __fadd_rn((float)(off + o), 0.5f)), -0.5f);
  return org + (int)fmaxf(s, 0.f);
}

// chroma terms of one (U,V) pair, shared by the pixels of a 2x2 block (R#11)
struct Chroma {
  int r, g, b;
};
__device__ __forceinline__ Chroma chroma(uint32_t uvpair) {
  const int u = (int)(uvpair & 0xffu) - 128;
  const int v = (int)((uvpair >> 8) & 0xffu) - 128;
  return {1673527 * v, -852492 * v - 409993 * u, 2116026 * u};
}
__device__ __forceinline__ int sat8(int x) { return min(max(x, 0), 255); }
// RGBx word: R | G << 8 | B << 16 | 0x4B << 24. The top byte is the exponent byte of 2^23,
// so a channel becomes the float 2^23 + value with one byte permute (see biased()).
__device__ __forceinline__ uint32_t rgbx(int Y, const Chroma& c) {
  const int yy = max(Y - 16, 0) * 1220542 + (1 << 19);
  return (uint32_t)sat8((yy + c.r) >> 20) | ((uint32_t)sat8((yy + c.g) >> 20) << 8) |
         ((uint32_t)sat8((yy + c.b) >> 20) << 16) | 0x4B000000u;
}

// byte C of an RGBx word as the float 2^23 + byte (exact): result bytes = [w.C, 0, 0, w.3]
template <int C>
__device__ __forceinline__ float biased(uint32_t w) {
  uint32_t r;
  asm("prmt.b32 %0, %1, 0, %2;" : "=r"(r) : "r"(w), "n"(0x3440 | C));
  return __uint_as_float(r);
}

// Packed fp32 pairs as 64-bit values (PTX f32x2 ops, sm_100a FFMA2/FADD2): the 64-bit type
// keeps each pair in an aligned register pair, so no MOVs are needed to feed the packed units.
// .rn ops are never contracted, so every op rounds exactly as the scalar R#12 sequence.
namespace f2 {
__device__ __forceinline__ uint64_t fma(uint64_t a, uint64_t b, uint64_t c) {
  uint64_t d;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
  return d;
}
__device__ __forceinline__ uint64_t add(uint64_t a, uint64_t b) {
  uint64_t d;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}
__device__ __forceinline__ uint64_t pack(uint32_t lo, uint32_t hi) {
  uint64_t d;
  asm("mov.b64 %0, {%1, %2};" : "=l"(d) : "r"(lo), "r"(hi));
  return d;
}
__device__ __forceinline__ uint64_t pack(float lo, float hi) { return pack(__float_as_uint(lo), __float_as_uint(hi)); }
__device__ __forceinline__ uint64_t splat(float x) { return pack(x, x); }
__device__ __forceinline__ uint32_t lo(uint64_t v) { return (uint32_t)v; }
__device__ __forceinline__ uint32_t hi(uint64_t v) { return (uint32_t)(v >> 32); }
__device__ __forceinline__ float lof(uint64_t v) { return __uint_as_float(lo(v)); }
__device__ __forceinline__ float hif(uint64_t v) { return __uint_as_float(hi(v)); }
}  // namespace f2

struct Row3 {
  uint64_t h[3];   // horizontal lerps of (column a, column b) per channel, packed fp32 pairs
};

template <int C>
__device__ __forceinline__ uint64_t hlerp(uint32_t a0, uint32_t a1, uint32_t b0, uint32_t b1, uint64_t lx) {
  const uint64_t P0 = f2::pack(__float_as_uint(biased<C>(a0)), __float_as_uint(biased<C>(b0)));
  const uint64_t P1 = f2::pack(__float_as_uint(biased<C>(a1)), __float_as_uint(biased<C>(b1)));
  const uint64_t d = f2::fma(P0, f2::splat(-1.f), P1);     // p1 - p0 (exact)
  const uint64_t p0 = f2::add(P0, f2::splat(-kBias));      // p0 (exact)
  return f2::fma(lx, d, p0);                               // fmaf(l, p1 - p0, p0)
}

// rint of a packed pair of values in [0, 256) as 1.5*2^23 + q (RNE); the low byte of each
// word is q
__device__ __forceinline__ uint64_t rint_biased(uint64_t v) { return f2::add(v, f2::splat(kRound)); }

__device__ __forceinline__ void hrow(Row3& r, const uint32_t* __restrict__ grow, uint32_t ca, uint32_t cb,
                                     uint64_t lx) {
  const uint32_t a0 = grow[ca & 0xffffu], a1 = grow[ca >> 16];
  const uint32_t b0 = grow[cb & 0xffffu], b1 = grow[cb >> 16];
  r.h[0] = hlerp<0>(a0, a1, b0, b1, lx);
  r.h[1] = hlerp<1>(a0, a1, b0, b1, lx);
  r.h[2] = hlerp<2>(a0, a1, b0, b1, lx);
}

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem) {
  const uint32_t s = (uint32_t)__cvta_generic_to_shared(smem);
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() {
  asm volatile("cp.async.commit_group;\ncp.async.wait_group 0;\n" ::: "memory");
}

// One destination (view k, time t, clip b) of the thread's two columns.
struct Dest {
  uint8_t* row;         // element (c=0, oy=current row, ox) of this destination
  uint32_t cstride;     // bytes between channel planes
  uint32_t rstride;     // bytes between rows
  float a[3], b[3];
};

__device__ __forceinline__ Dest make_dest(const LaunchParams& p, uint32_t dest, int oy, int ox) {
  const uint32_t k = dest >> 24, t = (dest >> 16) & 0xffu, b = dest & 0xffffu;
  const ViewConst& vc = p.views[k];
  Dest d;
  const size_t es = vc.dtype == SAND_U8 ? 1 : (vc.dtype == SAND_BF16 ? 2 : 4);
  const size_t plane = (size_t)vc.out_h * vc.out_w;
  d.cstride = (uint32_t)((size_t)vc.T * plane * es);
  d.rstride = (uint32_t)((size_t)vc.out_w * es);
  d.row = static_cast<uint8_t*>(p.out[k]) + ((((size_t)b * 3) * vc.T + t) * plane + (size_t)oy * vc.out_w + ox) * es;
#pragma unroll
  for (int c = 0; c < 3; ++c) {
    d.a[c] = vc.a[c];
    d.b[c] = vc.b[c];
  }
  return d;
}

// store quantised pair of channel c: q holds the integers 0..255 as floats, tq the same as
// 1.5*2^23 + q (low byte = q); DT < 0: dtype read at run time
template <int DT, bool VEC>
__device__ __forceinline__ void put(const Dest& d, int dtype, int c, uint64_t q, uint64_t tq, bool vec_rt, bool has_b) {
  const bool vec = VEC || vec_rt;
  const int dt = DT >= 0 ? DT : dtype;
  uint8_t* o = d.row + (size_t)c * d.cstride;
  if (dt == SAND_U8) {
    const uint32_t pair = __byte_perm(f2::lo(tq), f2::hi(tq), 0x0040);
    if (vec) {
      *reinterpret_cast<uint16_t*>(o) = (uint16_t)pair;
    } else {
      o[0] = (uint8_t)pair;
      if (has_b) o[1] = (uint8_t)(pair >> 8);
    }
    return;
  }
  // y = fmaf(q, a_c, b_c) per element (R#17)
  const uint64_t y = f2::fma(q, f2::splat(d.a[c]), f2::splat(d.b[c]));
  if (dt == SAND_BF16) {
    if (vec) {
      *reinterpret_cast<__nv_bfloat162*>(o) = __floats2bfloat162_rn(f2::lof(y), f2::hif(y));
    } else {
      reinterpret_cast<__nv_bfloat16*>(o)[0] = __float2bfloat16_rn(f2::lof(y));
      if (has_b) reinterpret_cast<__nv_bfloat16*>(o)[1] = __float2bfloat16_rn(f2::hif(y));
    }
  } else {
    if (vec) {
      *reinterpret_cast<uint64_t*>(o) = y;
    } else {
      reinterpret_cast<float*>(o)[0] = f2::lof(y);
      if (has_b) reinterpret_cast<float*>(o)[1] = f2::hif(y);
    }
  }
}

// Vertical lerp + rint + stores of one output row from the horizontal lerps of its two
// source rows (top = y0, bot = y1): v = fmaf(ly, h1 - h0, h0), q = rint(v) (R#12).
template <int DT, int ND, bool VEC>
__device__ __forceinline__ void emit(const Row3& top, const Row3& bot, float l, Dest (&dl)[ND], const int (&dt)[ND],
                                     const LaunchParams& p, const uint32_t* __restrict__ dests, int nd, int oy,
                                     int ox, bool vec, bool has_b) {
  const uint64_t ly = f2::splat(l);
  uint64_t q[3], tq[3];
#pragma unroll
  for (int c = 0; c < 3; ++c) {
    const uint64_t dv = f2::fma(top.h[c], f2::splat(-1.f), bot.h[c]);   // h1 - h0
    tq[c] = rint_biased(f2::fma(ly, dv, top.h[c]));                     // rint(fmaf(ly, h1-h0, h0))
    q[c] = DT == SAND_U8 ? tq[c] : f2::add(tq[c], f2::splat(-kRound));
  }
#pragma unroll
  for (int d = 0; d < ND; ++d) {
    if (d == 0 || d < nd) {
#pragma unroll
      for (int c = 0; c < 3; ++c) put<DT, VEC>(dl[d], dt[d], c, q[c], tq[c], vec, has_b);
      dl[d].row += dl[d].rstride;
    }
  }
  for (int d = ND; d < nd; ++d) {       // rare: more destinations than registers
    const Dest e = make_dest(p, dests[d], oy, ox);
    const int et = DT >= 0 ? DT : p.views[dests[d] >> 24].dtype;
#pragma unroll
    for (int c = 0; c < 3; ++c) put<DT, VEC>(e, et, c, q[c], tq[c], vec, has_b);
  }
}

// Walk band rows [rr_lo, rr_hi) for the output column pair (ox, ox+1). ND: destinations in
// registers (1, or 2 plus a loop over the rest). Horizontal lerps of source rows live in two
// register slots indexed by row parity: y1 = y0 + 1 (or y0 at the clamp), so the two rows an
// output row needs are always in different slots and each source row's lerp is computed
// once, with no register copies between rows (the branches on parity are warp-uniform).
template <int DT, int ND, bool VEC>
__device__ __forceinline__ void walk_rows(const LaunchParams& p, const uint32_t* __restrict__ dests, int nd,
                                          const uint2* __restrict__ rtab, const uint32_t* __restrict__ grid,
                                          int gw, int oy0, int rr_lo, int rr_hi, int ox, uint32_t ca, uint32_t cb,
                                          uint64_t lx, bool vec, bool has_b) {
  Dest dl[ND];
  int dt[ND];
#pragma unroll
  for (int d = 0; d < ND; ++d) {
    dl[d] = make_dest(p, dests[d], oy0 + rr_lo, ox);
    dt[d] = DT >= 0 ? DT : p.views[dests[d] >> 24].dtype;
  }
  int have0 = -1, have1 = -1;      // source row held in slot 0 (even rows) / slot 1 (odd rows)
  Row3 S0, S1;
  for (int rr = rr_lo; rr < rr_hi; ++rr) {
    const uint2 rt = rtab[rr];
    const int r0 = (int)(rt.x & 0xffffu), r1 = (int)(rt.x >> 16);
    const float l = __uint_as_float(rt.y);
    if (r0 & 1) {
      if (have1 != r0) { hrow(S1, grid + (size_t)r0 * gw, ca, cb, lx); have1 = r0; }
      if (r1 != r0) {
        if (have0 != r1) { hrow(S0, grid + (size_t)r1 * gw, ca, cb, lx); have0 = r1; }
        emit<DT, ND, VEC>(S1, S0, l, dl, dt, p, dests, nd, oy0 + rr, ox, vec, has_b);
      } else {
        emit<DT, ND, VEC>(S1, S1, l, dl, dt, p, dests, nd, oy0 + rr, ox, vec, has_b);
      }
    } else {
      if (have0 != r0) { hrow(S0, grid + (size_t)r0 * gw, ca, cb, lx); have0 = r0; }
      if (r1 != r0) {
        if (have1 != r1) { hrow(S1, grid + (size_t)r1 * gw, ca, cb, lx); have1 = r1; }
        emit<DT, ND, VEC>(S0, S1, l, dl, dt, p, dests, nd, oy0 + rr, ox, vec, has_b);
      } else {
        emit<DT, ND, VEC>(S0, S0, l, dl, dt, p, dests, nd, oy0 + rr, ox, vec, has_b);
      }
    }
  }
}

// The row walk (step 3), shared by both modes. grid: RGBx rows of gw words.
template <int DT, bool VEC>
__device__ __forceinline__ void walk(const LaunchParams& p, const WorkItem& w, const GroupParams& g,
                                     const Tables& t, const uint32_t* __restrict__ grid, int gw, int oy_lo,
                                     int nrows) {
  const int Wo = g.out_w;
  const int pairs = (Wo + 1) >> 1;
  const int P = blockDim.x >> 1;                       // threads per walker
  const int walker = threadIdx.x >= P ? 1 : 0;
  const int half = (nrows + 1) >> 1;
  const int rr_lo = walker * half, rr_hi = min(nrows, rr_lo + half);
  const int nd = (int)w.n_dest;
  const uint32_t* dests = p.dests + w.dest_begin;
  const uint2* rtab = reinterpret_cast<const uint2*>(t.rtab);
  for (int pair = threadIdx.x - walker * P; pair < pairs; pair += P) {
    const int ox = 2 * pair;
    const bool has_b = ox + 1 < Wo;
    const bool vec = has_b && !(Wo & 1);
    const int ja = g.flip ? Wo - 1 - ox : ox;
    const int jb = has_b ? (g.flip ? Wo - 2 - ox : ox + 1) : ja;
    const uint2 ta = t.ctab[ja], tb = t.ctab[jb];
    const uint64_t lx = f2::pack(ta.y, tb.y);
    if (nd == 1)
      walk_rows<DT, 1, VEC>(p, dests, nd, rtab, grid, gw, oy_lo, rr_lo, rr_hi, ox, ta.x, tb.x, lx, vec, has_b);
    else
      walk_rows<DT, kInlineDests, VEC>(p, dests, nd, rtab, grid, gw, oy_lo, rr_lo, rr_hi, ox, ta.x, tb.x, lx, vec,
                                  has_b);
  }
}

}  // namespace rs

// RAW mode: p launch params; R band rows; nbands; maxWo table sizing.
template <int DT, bool VEC>
__global__ void __launch_bounds__(224, 3) k_resample_raw(const LaunchParams p, int R, int nbands, int maxWo) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  using namespace rs;
  const int item_idx = blockIdx.x / nbands;
  const int band = blockIdx.x - item_idx * nbands;
  const WorkItem w = p.items[item_idx];
  if (w.flags & 1u) return;
  const GroupParams& g = p.groups[w.gp];
  const int Wo = g.out_w, Ho = g.out_h;
  const int oy_lo = band * R;
  if (oy_lo >= Ho) return;
  const int nrows = min(R, Ho - oy_lo);
  uint8_t* sp = smem_raw;
  const Tables t = carve_tables(sp, maxWo, R);
  const int tid = threadIdx.x, nthr = blockDim.x;

  // footprint: monotone taps -> first/last output column and row bound it
  const int x_lo = tap0(g.sc_x, g.off_x, 0, g.org_x);
  int x_hi, y_lo, y_hi, dmy;
  float fl;
  tap(g.sc_x, g.off_x, Wo - 1, g.lim_x, g.org_x, dmy, x_hi, fl);
  y_lo = tap0(g.sc_y, g.off_y, oy_lo, g.org_y);
  tap(g.sc_y, g.off_y, oy_lo + nrows - 1, g.lim_y, g.org_y, dmy, y_hi, fl);
  const int x16 = x_lo & ~15;
  const int gw = ((x_hi + 16) & ~15) - x16;        // grid / raw row width (bytes of Y, words of RGBx)
  const int ny = y_hi - y_lo + 1;
  const int uv_lo = y_lo >> 1;
  const int nuv = (y_hi >> 1) - uv_lo + 1;
  uint8_t* rawY = sp;
  uint8_t* rawUV = rawY + (size_t)ny * gw;
  uint32_t* grid = reinterpret_cast<uint32_t*>(rawUV + a16((size_t)nuv * gw));

  // 1. async copy of the NV12 footprint (16 B requests)
  const uint8_t* Yp = p.slab + w.y_off;
  const uint8_t* UVp = Yp + (size_t)w.pitch * w.src_h;
  const int chunks = gw >> 4;
  {
    // thread -> (row slot, chunk): rows advance by nthr / chunks per pass, no division in the loop
    const int rows_per_pass = max(1, nthr / chunks);
    const int k = tid % chunks, r0 = tid / chunks;
    if (r0 < rows_per_pass)
      for (int r = r0; r < ny + nuv; r += rows_per_pass) {
        if (r < ny)
          cp_async16(rawY + (size_t)r * gw + k * 16, Yp + (size_t)(y_lo + r) * w.pitch + x16 + k * 16);
        else
          cp_async16(rawUV + (size_t)(r - ny) * gw + k * 16, UVp + (size_t)(uv_lo + r - ny) * w.pitch + x16 + k * 16);
      }
    for (int kk = k + nthr; kk < chunks; kk += nthr)     // only if a row has more chunks than threads
      for (int r = 0; r < ny + nuv; ++r) {
        if (r < ny)
          cp_async16(rawY + (size_t)r * gw + kk * 16, Yp + (size_t)(y_lo + r) * w.pitch + x16 + kk * 16);
        else
          cp_async16(rawUV + (size_t)(r - ny) * gw + kk * 16, UVp + (size_t)(uv_lo + r - ny) * w.pitch + x16 + kk * 16);
      }
  }
  // 2. tap tables, grid-relative (overlaps the copy)
  for (int j = tid; j < Wo; j += nthr) {
    int x0, x1;
    float lx;
    tap(g.sc_x, g.off_x, j, g.lim_x, g.org_x, x0, x1, lx);
    t.ctab[j] = make_uint2((uint32_t)(x0 - x16) | ((uint32_t)(x1 - x16) << 16), __float_as_uint(lx));
  }
  for (int r = tid; r < nrows; r += nthr) {
    int y0, y1;
    float ly;
    tap(g.sc_y, g.off_y, oy_lo + r, g.lim_y, g.org_y, y0, y1, ly);
    t.rtab[r] = make_uint2((uint32_t)(y0 - y_lo) | ((uint32_t)(y1 - y_lo) << 16), __float_as_uint(ly));
  }
  cp_async_wait_all();
  __syncthreads();

  // 3. NV12 -> RGBx in shared memory: a thread takes one chroma sample and the (up to) 2x2
  //    luma pixels that share it; warps walk chroma rows, lanes walk chroma columns
  const int hp = gw >> 1;
  const int nwarps = nthr >> 5, lane = tid & 31;
  for (int u = tid >> 5; u < nuv; u += nwarps) {
    const int ytop = 2 * (uv_lo + u) - y_lo;      // grid rows ytop, ytop+1 (may fall outside)
    const bool top = ytop >= 0, bot = ytop + 1 < ny;
    const uint8_t* uvrow = rawUV + (size_t)u * gw;
    for (int k = lane; k < hp; k += 32) {
      const Chroma ch = chroma(*reinterpret_cast<const uint16_t*>(uvrow + 2 * k));
      if (top) {
        const uint32_t yp = *reinterpret_cast<const uint16_t*>(rawY + (size_t)ytop * gw + 2 * k);
        *reinterpret_cast<uint2*>(grid + (size_t)ytop * gw + 2 * k) =
            make_uint2(rgbx((int)(yp & 0xffu), ch), rgbx((int)(yp >> 8), ch));
      }
      if (bot) {
        const uint32_t yp = *reinterpret_cast<const uint16_t*>(rawY + (size_t)(ytop + 1) * gw + 2 * k);
        *reinterpret_cast<uint2*>(grid + (size_t)(ytop + 1) * gw + 2 * k) =
            make_uint2(rgbx((int)(yp & 0xffu), ch), rgbx((int)(yp >> 8), ch));
      }
    }
  }
  __syncthreads();

  // 4. row walk
  walk<DT, VEC>(p, w, g, t, grid, gw, oy_lo, nrows);
}

// GATHER mode (heavy down-scaling): compact tap grid gathered from HBM.
template <int DT, bool VEC>
__global__ void __launch_bounds__(224, 3) k_resample_gather(const LaunchParams p, int R, int nbands, int maxWo) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  using namespace rs;
  const int item_idx = blockIdx.x / nbands;
  const int band = blockIdx.x - item_idx * nbands;
  const WorkItem w = p.items[item_idx];
  if (w.flags & 1u) return;
  const GroupParams& g = p.groups[w.gp];
  const int Wo = g.out_w, Ho = g.out_h;
  const int oy_lo = band * R;
  if (oy_lo >= Ho) return;
  const int nrows = min(R, Ho - oy_lo);
  uint8_t* sp = smem_raw;
  const Tables t = carve_tables(sp, maxWo, R);
  uint32_t* colbits = reinterpret_cast<uint32_t*>(sp); sp += a16(kColWords * 4);
  uint32_t* rowbits = reinterpret_cast<uint32_t*>(sp); sp += a16(kRowWords * 4);
  uint16_t* colpref = reinterpret_cast<uint16_t*>(sp); sp += a16(kColWords * 2);
  uint16_t* rowpref = reinterpret_cast<uint16_t*>(sp); sp += a16(kRowWords * 2);
  uint16_t* xs = reinterpret_cast<uint16_t*>(sp); sp += a16((size_t)2 * maxWo * 2);
  uint16_t* ys = reinterpret_cast<uint16_t*>(sp); sp += a16((size_t)2 * R * 2);
  uint32_t* grid = reinterpret_cast<uint32_t*>(sp);
  const int tid = threadIdx.x, nthr = blockDim.x;
  const int warp = tid >> 5, lane = tid & 31;

  for (int i = tid; i < kColWords + kRowWords; i += nthr) {
    if (i < kColWords) colbits[i] = 0u;
    else rowbits[i - kColWords] = 0u;
  }
  const int cbase = tap0(g.sc_x, g.off_x, 0, g.org_x);
  const int rbase = tap0(g.sc_y, g.off_y, oy_lo, g.org_y);
  __syncthreads();
  for (int j = tid; j < Wo; j += nthr) {
    int x0, x1;
    float lx;
    tap(g.sc_x, g.off_x, j, g.lim_x, g.org_x, x0, x1, lx);
    const int r0 = x0 - cbase, r1 = x1 - cbase;
    t.ctab[j] = make_uint2((uint32_t)r0 | ((uint32_t)r1 << 16), __float_as_uint(lx));
    atomicOr(&colbits[r0 >> 5], 1u << (r0 & 31));
    atomicOr(&colbits[r1 >> 5], 1u << (r1 & 31));
  }
  for (int r = tid; r < nrows; r += nthr) {
    int y0, y1;
    float ly;
    tap(g.sc_y, g.off_y, oy_lo + r, g.lim_y, g.org_y, y0, y1, ly);
    const int r0 = y0 - rbase, r1 = y1 - rbase;
    t.rtab[r] = make_uint2((uint32_t)r0 | ((uint32_t)r1 << 16), __float_as_uint(ly));
    atomicOr(&rowbits[r0 >> 5], 1u << (r0 & 31));
    atomicOr(&rowbits[r1 >> 5], 1u << (r1 & 31));
  }
  __syncthreads();
  if (warp == 0) {   // exclusive popcount prefix of the column bitmap
    uint32_t c[kColWords / 32];
    uint32_t sum = 0;
#pragma unroll
    for (int k = 0; k < kColWords / 32; ++k) {
      c[k] = __popc(colbits[lane * (kColWords / 32) + k]);
      sum += c[k];
    }
    uint32_t incl = sum;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t o = __shfl_up_sync(0xffffffffu, incl, d);
      if (lane >= d) incl += o;
    }
    uint32_t run = incl - sum;
#pragma unroll
    for (int k = 0; k < kColWords / 32; ++k) {
      colpref[lane * (kColWords / 32) + k] = (uint16_t)run;
      run += c[k];
    }
    if (lane == 31) t.misc[0] = (int)incl;
  }
  if (warp == (nthr > 32 ? 1 : 0)) {   // ... and of the row bitmap
    const uint32_t c = __popc(rowbits[lane]);
    uint32_t incl = c;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t o = __shfl_up_sync(0xffffffffu, incl, d);
      if (lane >= d) incl += o;
    }
    rowpref[lane] = (uint16_t)(incl - c);
    if (lane == 31) t.misc[1] = (int)incl;
  }
  __syncthreads();
  for (int wd = tid; wd < kColWords + kRowWords; wd += nthr) {
    const bool col = wd < kColWords;
    const int k0 = col ? wd : wd - kColWords;
    uint32_t b = col ? colbits[k0] : rowbits[k0];
    int k = col ? colpref[k0] : rowpref[k0];
    const int base = (col ? cbase : rbase) + k0 * 32;
    uint16_t* dst = col ? xs : ys;
    while (b) {
      const int bit = __ffs(b) - 1;
      b &= b - 1;
      dst[k++] = (uint16_t)(base + bit);
    }
  }
  auto cidx = [&](const uint32_t* bits, const uint16_t* pref, int r) -> uint32_t {
    return pref[r >> 5] + __popc(bits[r >> 5] & ((1u << (r & 31)) - 1u));
  };
  for (int j = tid; j < Wo; j += nthr) {
    const uint32_t v = t.ctab[j].x;
    t.ctab[j].x = cidx(colbits, colpref, (int)(v & 0xffffu)) | (cidx(colbits, colpref, (int)(v >> 16)) << 16);
  }
  for (int r = tid; r < nrows; r += nthr) {
    const uint32_t v = t.rtab[r].x;
    t.rtab[r].x = cidx(rowbits, rowpref, (int)(v & 0xffffu)) | (cidx(rowbits, rowpref, (int)(v >> 16)) << 16);
  }
  __syncthreads();

  // gather-convert with 4 independent loads in flight per thread
  const int nX = t.misc[0], nY = t.misc[1];
  const uint8_t* Yp = p.slab + w.y_off;
  const uint8_t* UVp = Yp + (size_t)w.pitch * w.src_h;
  const int nwarps = nthr >> 5;
  for (int i = warp; i < nY; i += nwarps) {
    const int y = ys[i];
    const uint8_t* yrow = Yp + (size_t)y * w.pitch;
    const uint8_t* uvrow = UVp + (size_t)(y >> 1) * w.pitch;
    uint32_t* grow = grid + (size_t)i * nX;
    for (int j0 = lane; j0 < nX; j0 += 128) {
      int yv[4];
      uint32_t uvv[4];
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int jj = j0 + 32 * u;
        if (jj < nX) {
          const int x = xs[jj];
          yv[u] = __ldg(yrow + x);
          uvv[u] = __ldg(reinterpret_cast<const uint16_t*>(uvrow + (x & ~1)));
        }
      }
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const int jj = j0 + 32 * u;
        if (jj < nX) grow[jj] = rgbx(yv[u], chroma(uvv[u]));
      }
    }
  }
  __syncthreads();
  walk<DT, VEC>(p, w, g, t, grid, nX, oy_lo, nrows);
}

}  // namespace sand
