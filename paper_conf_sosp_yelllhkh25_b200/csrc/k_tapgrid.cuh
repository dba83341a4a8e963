// k_tapgrid.cuh — v2 fused resample kernel for items without rotation/blur
// (DESIGN.md §7 "tap-grid kernel").
//
// One CTA = one work item (clip slot, source frame, group) x one band of R output rows.
//  1. Separable tap tables: output column j -> source taps (x0, x1, lambda_x); output row
//     -> (y0, y1, lambda_y) (R#12, exact fp32 rule).
//  2. Tap grid: the distinct tapped source columns Xs and rows Ys of the band (bitmaps +
//     popcount prefix). For up-/mild down-scaling this is the whole crop footprint; for
//     heavy down-scaling (1080p -> 224) only the tapped lines are touched (a4).
//  3. Gather-convert: every grid pixel is read once from the NV12 frame (coalesced along
//     rows) and converted to RGB (a5, Q1) into shared memory as packed RGBx words.
//  4. Two row-walker groups; each thread owns two adjacent output columns and walks down
//     its half of the band keeping the horizontal lerps of the two current source rows in
//     registers, so each (source row, column) lerp is computed once (a6). Flip is the
//     column mirror (a7). Vertical lerp, rint, normalise and bf16 packing run on
//     FFMA2/FADD2 pairs (sm_100a packed fp32), then one 4-byte store per (row, channel,
//     destination) (a10); every destination view of the group is written from the same
//     registers (a11).
// All fp32 arithmetic is the R#12/R#17 op sequence with IEEE rounding at each step, so the
// result is bit-identical to the oracle (byte->float via the 2^23 exponent trick and rint via
// +1.5*2^23 are exact for values in [0, 256)).
#pragma once

namespace sand {
namespace tg {

constexpr int kColWords = 128;   // source column span <= 4096
constexpr int kRowWords = 32;    // band source row span <= 1024
constexpr float kBias = 8388608.0f;        // 2^23
constexpr float kRound = 12582912.0f;      // 1.5 * 2^23

struct Smem {
  uint32_t* colbits;
  uint32_t* rowbits;
  uint16_t* colpref;
  uint16_t* rowpref;
  uint32_t* ctab_i;   // per output column j: (ci0 | ci1 << 16), later compact grid indices
  float* ctab_l;
  uint32_t* rtab_i;   // per band row
  float* rtab_l;
  uint16_t* xs;       // compact column -> source column
  uint16_t* ys;       // compact row -> source row
  int* counts;        // [0] = nXs, [1] = nYs
  uint32_t* grid;     // RGBx [nYs][nXs]
};

__host__ __device__ inline size_t align16(size_t x) { return (x + 15) & ~size_t(15); }

// bytes of the table part of the shared layout for output width maxWo and band R
__host__ __device__ inline size_t table_bytes(int maxWo, int R) {
  size_t b = 0;
  b += align16(kColWords * 4) + align16(kRowWords * 4);
  b += align16(kColWords * 2) + align16(kRowWords * 2);
  b += align16((size_t)maxWo * 4) * 2 + align16((size_t)R * 4) * 2;
  b += align16((size_t)2 * maxWo * 2) + align16((size_t)2 * R * 2);
  b += 16;
  return b;
}

__device__ inline Smem carve(uint8_t* base, int maxWo, int R) {
  Smem s;
  uint8_t* p = base;
  s.colbits = reinterpret_cast<uint32_t*>(p); p += align16(kColWords * 4);
  s.rowbits = reinterpret_cast<uint32_t*>(p); p += align16(kRowWords * 4);
  s.colpref = reinterpret_cast<uint16_t*>(p); p += align16(kColWords * 2);
  s.rowpref = reinterpret_cast<uint16_t*>(p); p += align16(kRowWords * 2);
  s.ctab_i = reinterpret_cast<uint32_t*>(p); p += align16((size_t)maxWo * 4);
  s.ctab_l = reinterpret_cast<float*>(p); p += align16((size_t)maxWo * 4);
  s.rtab_i = reinterpret_cast<uint32_t*>(p); p += align16((size_t)R * 4);
  s.rtab_l = reinterpret_cast<float*>(p); p += align16((size_t)R * 4);
  s.xs = reinterpret_cast<uint16_t*>(p); p += align16((size_t)2 * maxWo * 2);
  s.ys = reinterpret_cast<uint16_t*>(p); p += align16((size_t)2 * R * 2);
  s.counts = reinterpret_cast<int*>(p); p += 16;
  s.grid = reinterpret_cast<uint32_t*>(p);
  return s;
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

__device__ __forceinline__ uint32_t compact_index(const uint32_t* bits, const uint16_t* pref, int r) {
  return pref[r >> 5] + __popc(bits[r >> 5] & ((1u << (r & 31)) - 1u));
}

// NV12 -> packed RGBx (R#11, OpenCV integer BT.601)
__device__ __forceinline__ uint32_t rgbx(int Y, uint32_t uvpair) {
  const int u = (int)(uvpair & 0xffu) - 128;
  const int v = (int)(uvpair >> 8) - 128;
  const int yy = max(Y - 16, 0) * 1220542 + (1 << 19);
  const int R = min(max((yy + 1673527 * v) >> 20, 0), 255);
  const int G = min(max((yy - 852492 * v - 409993 * u) >> 20, 0), 255);
  const int B = min(max((yy + 2116026 * u) >> 20, 0), 255);
  return (uint32_t)R | ((uint32_t)G << 8) | ((uint32_t)B << 16);
}

// byte c of an RGBx word as the float 2^23 + byte (exact)
__device__ __forceinline__ float biased(uint32_t w, int c) {
  return __int_as_float((int)__byte_perm(w, 0x4B000000u, 0x7540u | (uint32_t)c));
}

struct Row3 {
  float2 h[3];   // horizontal lerps of (column a, column b) per channel
};

__device__ __forceinline__ Row3 hrow(const uint32_t* __restrict__ grow, uint32_t ca, uint32_t cb, float2 lx) {
  const uint32_t a0 = grow[ca & 0xffffu], a1 = grow[ca >> 16];
  const uint32_t b0 = grow[cb & 0xffffu], b1 = grow[cb >> 16];
  Row3 r;
#pragma unroll
  for (int c = 0; c < 3; ++c) {
    const float2 P0 = make_float2(biased(a0, c), biased(b0, c));
    const float2 P1 = make_float2(biased(a1, c), biased(b1, c));
    const float2 d = __ffma2_rn(P0, make_float2(-1.f, -1.f), P1);          // p1 - p0 (exact)
    const float2 p0 = __fadd2_rn(P0, make_float2(-kBias, -kBias));          // p0 (exact)
    r.h[c] = __ffma2_rn(lx, d, p0);                                         // fmaf(l, p1 - p0, p0)
  }
  return r;
}

// stores output columns (ox, ox+1) of one row/channel; `vec`: both columns valid and the pair
// is 2-element aligned (out_w even); otherwise column a and (if has_b) column b separately.
__device__ __forceinline__ void store_pair(const LaunchParams& p, uint32_t dest, int c, int oy, int ox,
                                           bool vec, bool has_b, float2 q) {
  const uint32_t k = dest >> 24, t = (dest >> 16) & 0xffu, b = dest & 0xffffu;
  const ViewConst& vc = p.views[k];
  const size_t idx = (((size_t)b * 3 + c) * vc.T + t) * ((size_t)vc.out_h * vc.out_w) + (size_t)oy * vc.out_w + ox;
  if (vc.dtype == SAND_BF16) {
    const float2 y = __ffma2_rn(q, make_float2(vc.a[c], vc.a[c]), make_float2(vc.b[c], vc.b[c]));
    __nv_bfloat16* o = static_cast<__nv_bfloat16*>(p.out[k]) + idx;
    if (vec) {
      *reinterpret_cast<__nv_bfloat162*>(o) = __floats2bfloat162_rn(y.x, y.y);
    } else {
      o[0] = __float2bfloat16_rn(y.x);
      if (has_b) o[1] = __float2bfloat16_rn(y.y);
    }
  } else if (vc.dtype == SAND_F32) {
    const float2 y = __ffma2_rn(q, make_float2(vc.a[c], vc.a[c]), make_float2(vc.b[c], vc.b[c]));
    float* o = static_cast<float*>(p.out[k]) + idx;
    if (vec) {
      *reinterpret_cast<float2*>(o) = y;
    } else {
      o[0] = y.x;
      if (has_b) o[1] = y.y;
    }
  } else {
    uint8_t* o = static_cast<uint8_t*>(p.out[k]) + idx;
    if (vec) {
      *reinterpret_cast<uint16_t*>(o) = (uint16_t)((uint32_t)q.x | ((uint32_t)q.y << 8));
    } else {
      o[0] = (uint8_t)q.x;
      if (has_b) o[1] = (uint8_t)q.y;
    }
  }
}

}  // namespace tg

// p: launch params; R: output rows per band; nbands = ceil(maxHo / R); maxWo: table sizing.
__global__ void __launch_bounds__(256, 2) k_tapgrid(const LaunchParams p, int R, int nbands, int maxWo) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  using namespace tg;
  const int item_idx = blockIdx.x / nbands;
  const int band = blockIdx.x - item_idx * nbands;
  const WorkItem w = p.items[item_idx];
  if (w.flags & 1u) return;
  const GroupParams& g = p.groups[w.gp];
  const int Wo = g.out_w, Ho = g.out_h;
  const int oy_lo = band * R;
  if (oy_lo >= Ho) return;
  const int nrows = min(R, Ho - oy_lo);
  Smem s = carve(smem_raw, maxWo, R);
  const int tid = threadIdx.x, nthr = blockDim.x;

  for (int i = tid; i < kColWords + kRowWords; i += nthr) {
    if (i < kColWords) s.colbits[i] = 0u;
    else s.rowbits[i - kColWords] = 0u;
  }
  int cbase, rbase, dummy;
  float fl;
  tap(g.sc_x, g.off_x, 0, g.lim_x, g.org_x, cbase, dummy, fl);
  tap(g.sc_y, g.off_y, oy_lo, g.lim_y, g.org_y, rbase, dummy, fl);
  __syncthreads();

  // 1. tap tables + bitmaps of tapped columns / rows
  for (int j = tid; j < Wo; j += nthr) {
    int x0, x1;
    float lx;
    tap(g.sc_x, g.off_x, j, g.lim_x, g.org_x, x0, x1, lx);
    const int r0 = x0 - cbase, r1 = x1 - cbase;
    s.ctab_i[j] = (uint32_t)r0 | ((uint32_t)r1 << 16);
    s.ctab_l[j] = lx;
    atomicOr(&s.colbits[r0 >> 5], 1u << (r0 & 31));
    atomicOr(&s.colbits[r1 >> 5], 1u << (r1 & 31));
  }
  for (int r = tid; r < nrows; r += nthr) {
    int y0, y1;
    float ly;
    tap(g.sc_y, g.off_y, oy_lo + r, g.lim_y, g.org_y, y0, y1, ly);
    const int r0 = y0 - rbase, r1 = y1 - rbase;
    s.rtab_i[r] = (uint32_t)r0 | ((uint32_t)r1 << 16);
    s.rtab_l[r] = ly;
    atomicOr(&s.rowbits[r0 >> 5], 1u << (r0 & 31));
    atomicOr(&s.rowbits[r1 >> 5], 1u << (r1 & 31));
  }
  __syncthreads();

  // 2. exclusive popcount prefix over the bitmaps (warp 0: columns, warp 1 or 0: rows)
  const int warp = tid >> 5, lane = tid & 31;
  if (warp == 0) {
    uint32_t c[kColWords / 32];
    uint32_t sum = 0;
#pragma unroll
    for (int k = 0; k < kColWords / 32; ++k) {
      c[k] = __popc(s.colbits[lane * (kColWords / 32) + k]);
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
      s.colpref[lane * (kColWords / 32) + k] = (uint16_t)run;
      run += c[k];
    }
    if (lane == 31) s.counts[0] = (int)incl;
  }
  if (warp == (nthr > 32 ? 1 : 0)) {
    const uint32_t c = __popc(s.rowbits[lane]);
    uint32_t incl = c;
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
      const uint32_t o = __shfl_up_sync(0xffffffffu, incl, d);
      if (lane >= d) incl += o;
    }
    s.rowpref[lane] = (uint16_t)(incl - c);
    if (lane == 31) s.counts[1] = (int)incl;
  }
  __syncthreads();

  // 3. compact lists and compact tap indices
  for (int wd = tid; wd < kColWords + kRowWords; wd += nthr) {
    if (wd < kColWords) {
      uint32_t b = s.colbits[wd];
      int k = s.colpref[wd];
      while (b) {
        const int bit = __ffs(b) - 1;
        b &= b - 1;
        s.xs[k++] = (uint16_t)(cbase + wd * 32 + bit);
      }
    } else {
      const int rw = wd - kColWords;
      uint32_t b = s.rowbits[rw];
      int k = s.rowpref[rw];
      while (b) {
        const int bit = __ffs(b) - 1;
        b &= b - 1;
        s.ys[k++] = (uint16_t)(rbase + rw * 32 + bit);
      }
    }
  }
  for (int j = tid; j < Wo; j += nthr) {
    const uint32_t v = s.ctab_i[j];
    s.ctab_i[j] = compact_index(s.colbits, s.colpref, (int)(v & 0xffffu)) |
                  (compact_index(s.colbits, s.colpref, (int)(v >> 16)) << 16);
  }
  for (int r = tid; r < nrows; r += nthr) {
    const uint32_t v = s.rtab_i[r];
    s.rtab_i[r] = compact_index(s.rowbits, s.rowpref, (int)(v & 0xffffu)) |
                  (compact_index(s.rowbits, s.rowpref, (int)(v >> 16)) << 16);
  }
  __syncthreads();

  // 4. gather-convert the tap grid (one read of each tapped NV12 pixel, coalesced along rows)
  const int nX = s.counts[0], nY = s.counts[1];
  const uint8_t* Yp = p.slab + w.y_off;
  const uint8_t* UVp = Yp + (size_t)w.pitch * w.src_h;
  const int nwarps = nthr >> 5;
  for (int i = warp; i < nY; i += nwarps) {
    const int y = s.ys[i];
    const uint8_t* yrow = Yp + (size_t)y * w.pitch;
    const uint8_t* uvrow = UVp + (size_t)(y >> 1) * w.pitch;
    uint32_t* grow = s.grid + (size_t)i * nX;
    for (int jj = lane; jj < nX; jj += 32) {
      const int x = s.xs[jj];
      const int Yv = __ldg(yrow + x);
      const uint32_t uv = __ldg(reinterpret_cast<const uint16_t*>(uvrow + (x & ~1)));
      grow[jj] = rgbx(Yv, uv);
    }
  }
  __syncthreads();

  // 5. row walkers: two groups, each thread owns output columns (2m, 2m+1)
  const int pairs = (Wo + 1) >> 1;
  const int walker = tid / pairs;
  if (walker >= 2) return;
  const int pair = tid - walker * pairs;
  const int ox = 2 * pair;
  const bool has_b = ox + 1 < Wo;
  const bool vec = has_b && !(Wo & 1);
  const int ja = g.flip ? Wo - 1 - ox : ox;
  const int jb = has_b ? (g.flip ? Wo - 2 - ox : ox + 1) : ja;
  const uint32_t ca = s.ctab_i[ja], cb = s.ctab_i[jb];
  const float2 lx = make_float2(s.ctab_l[ja], s.ctab_l[jb]);
  const int half = (nrows + 1) >> 1;
  const int rr_lo = walker * half, rr_hi = min(nrows, rr_lo + half);
  int ra = -1, rb = -1;
  Row3 Ha, Hb;
  const uint32_t* dests = p.dests + w.dest_begin;
  const int nd = (int)w.n_dest;
  for (int rr = rr_lo; rr < rr_hi; ++rr) {
    const uint32_t rt = s.rtab_i[rr];
    const int r0 = (int)(rt & 0xffffu), r1 = (int)(rt >> 16);
    const float ly1 = s.rtab_l[rr];
    Row3 H0, H1;
    if (r0 == rb) H0 = Hb;
    else if (r0 == ra) H0 = Ha;
    else H0 = hrow(s.grid + (size_t)r0 * nX, ca, cb, lx);
    if (r1 == r0) H1 = H0;
    else if (r1 == rb) H1 = Hb;
    else H1 = hrow(s.grid + (size_t)r1 * nX, ca, cb, lx);
    ra = r0; Ha = H0;
    rb = r1; Hb = H1;
    const float2 ly = make_float2(ly1, ly1);
    float2 q[3];
#pragma unroll
    for (int c = 0; c < 3; ++c) {
      const float2 dv = __ffma2_rn(H0.h[c], make_float2(-1.f, -1.f), H1.h[c]);   // h1 - h0
      const float2 v = __ffma2_rn(ly, dv, H0.h[c]);                              // fmaf(ly, h1-h0, h0)
      const float2 t = __fadd2_rn(v, make_float2(kRound, kRound));               // rint (RNE)
      q[c] = __fadd2_rn(t, make_float2(-kRound, -kRound));
    }
    const int oy = oy_lo + rr;
    for (int d = 0; d < nd; ++d) {
      const uint32_t dest = dests[d];
#pragma unroll
      for (int c = 0; c < 3; ++c) store_pair(p, dest, c, oy, ox, vec, has_b, q[c]);
    }
  }
}

}  // namespace sand
