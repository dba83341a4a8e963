// k_stencil.cuh — fused kernel for items with rotation and/or blur (two-view config;
// SURVEY §8(a) a4-a10).
//
// One CTA (512 threads, 227 KB shared memory: three uint8 Q2 planes + an 80 KB band/ring/
// scratch region) per stencil work item:
//  Phase 1  Q2 = resample(+flip) of the clip frame for all three channels into the planes,
//           band by band: cp.async of the band's NV12 rows (the next band's rows load while
//           this band is walked), conversion to an RGBx tap grid, column-pair walkers
//           writing uint8 (a4-a7, Q2).
//  Phase 2  rotation without blur: Q3 straight to the output (rotate_direct: rint, normalise,
//           store; a8, a10). Rotation then blur: Q3 in place through a power-of-two ring of
//           rows (rotate_inplace). Blur (a9), channel by channel, last to first so finished
//           planes extend the fp32 strip scratch: horizontal pass in kBX-column register
//           blocks over row pairs (compile-time reflect maps for the border blocks), vertical
//           pass in kBV-row blocks over column pairs, rint (Q4), normalise, pair stores.
// Every fp32 operation follows R#12/R#15/R#16/R#17 with IEEE rounding in the oracle's order
// (blur taps accumulated from 0 in tap order), so outputs are bit-identical to the oracle.
#pragma once

namespace sand {
namespace sc {

using rs::a16;

struct Shape {
  int R;            // Q2 band height (output rows)
  int gw;           // max grid row width (bytes of Y / words of RGBx)
  int grid_rows;    // grid / raw capacity in rows per band
  size_t plane;     // bytes of one uint8 plane (Ho*Wo, 16-aligned)
  size_t ubytes;    // bytes of the shared band/Q3 region
};

__host__ __device__ inline size_t band_bytes(int maxWo, int R, int grid_rows, int gw) {
  return a16((size_t)maxWo * 8) + a16((size_t)R * 16) + (size_t)grid_rows * gw * 4 + a16((size_t)(grid_rows + grid_rows / 2 + 2) * gw);
}

__device__ __forceinline__ uint32_t ldsu8(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ void stsu8(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u8 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void stsu16(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u16 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void sts32(uint32_t a, uint32_t v) {
  asm volatile("st.shared.u32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ __forceinline__ void sts64f(uint32_t a, float2 v) {
  asm volatile("st.shared.v2.f32 [%0], {%1, %2};" ::"r"(a), "f"(v.x), "f"(v.y) : "memory");
}
__device__ __forceinline__ float2 lds64f(uint32_t a) {
  float2 v;
  asm volatile("ld.shared.v2.f32 {%0, %1}, [%2];" : "=f"(v.x), "=f"(v.y) : "r"(a));
  return v;
}
__device__ __forceinline__ float u8f(uint32_t b) {    // exact float of a byte
  return __fadd_rn(__uint_as_float(0x4B000000u | b), -rs::kBias);
}
__device__ __forceinline__ int reflect(int i, int n) { return i < 0 ? -i : (i >= n ? 2 * (n - 1) - i : i); }

// destination base pointer of channel c for dest entry `dest` (element (0, 0) of the plane)
__device__ __forceinline__ uint8_t* plane_ptr(const LaunchParams& p, uint32_t dest, int c, size_t& es) {
  const uint32_t k = dest >> 24, t = (dest >> 16) & 0xffu, b = dest & 0xffffu;
  const ViewConst& vc = p.views[k];
  es = vc.dtype == SAND_U8 ? 1 : (vc.dtype == SAND_BF16 ? 2 : 4);
  const size_t plane = (size_t)vc.out_h * vc.out_w;
  return static_cast<uint8_t*>(p.out[k]) + (((size_t)b * 3 + c) * vc.T + t) * plane * es;
}

// one destination plane (view, clip, t, channel) with its normalisation constants (R#17)
struct ChDest {
  uint8_t* base;     // element (0, 0) of the plane
  float a, b;
  int dt, es;
};

__device__ __forceinline__ ChDest ch_dest(const LaunchParams& p, uint32_t dest, int c) {
  const ViewConst& vc = p.views[dest >> 24];
  size_t es;
  ChDest d;
  d.base = plane_ptr(p, dest, c, es);
  d.es = (int)es;
  d.dt = vc.dtype;
  d.a = vc.a[c];
  d.b = vc.b[c];
  return d;
}

template <int DT, bool VEC>
__device__ __forceinline__ void put_q(const ChDest& d, int oy, int ox, int Wo, float2 q, bool has_b) {
  const bool vec = VEC || (has_b && !(Wo & 1));
  const int dt = DT >= 0 ? DT : d.dt;
  const int es = DT >= 0 ? (DT == SAND_U8 ? 1 : (DT == SAND_BF16 ? 2 : 4)) : d.es;
  uint8_t* o = d.base + (size_t)(oy * Wo + ox) * es;
  if (dt == SAND_BF16) {
    const float2 y = __ffma2_rn(q, make_float2(d.a, d.a), make_float2(d.b, d.b));
    if (vec) {
      *reinterpret_cast<__nv_bfloat162*>(o) = __floats2bfloat162_rn(y.x, y.y);
    } else {
      reinterpret_cast<__nv_bfloat16*>(o)[0] = __float2bfloat16_rn(y.x);
      if (has_b) reinterpret_cast<__nv_bfloat16*>(o)[1] = __float2bfloat16_rn(y.y);
    }
  } else if (dt == SAND_F32) {
    const float2 y = __ffma2_rn(q, make_float2(d.a, d.a), make_float2(d.b, d.b));
    if (vec) {
      *reinterpret_cast<float2*>(o) = y;
    } else {
      reinterpret_cast<float*>(o)[0] = y.x;
      if (has_b) reinterpret_cast<float*>(o)[1] = y.y;
    }
  } else {
    if (vec) {
      *reinterpret_cast<uint16_t*>(o) = (uint16_t)((uint32_t)q.x | ((uint32_t)q.y << 8));
    } else {
      o[0] = (uint8_t)q.x;
      if (has_b) o[1] = (uint8_t)q.y;
    }
  }
}

// the destinations of one channel: two in registers, the rest recomputed (rare)
struct ChDests {
  ChDest d0, d1;
  int nd;
  const uint32_t* dests;
  int c;
};

template <int DT, bool VEC>
__device__ __forceinline__ void store_q(const LaunchParams& p, const ChDests& cd, int oy, int ox, int Wo, float2 q,
                                        bool has_b) {
  put_q<DT, VEC>(cd.d0, oy, ox, Wo, q, has_b);
  if (cd.nd > 1) put_q<DT, VEC>(cd.d1, oy, ox, Wo, q, has_b);
  for (int d = 2; d < cd.nd; ++d) put_q<DT, VEC>(ch_dest(p, cd.dests[d], cd.c), oy, ox, Wo, q, has_b);
}

// q pair (biased: 1.5*2^23 + q per lane, the rint result) -> normalise (R#17) -> one 2-element
// store at o (compile-time dtype, aligned pair)
template <int DT>
__device__ __forceinline__ void put_pair(uint8_t* o, uint64_t tq, uint64_t na, uint64_t nb) {
  using namespace rs;
  if constexpr (DT == SAND_U8) {
    *reinterpret_cast<uint16_t*>(o) = (uint16_t)__byte_perm(f2::lo(tq), f2::hi(tq), 0x0040);
  } else {
    const uint64_t y = f2::fma(f2::add(tq, f2::splat(-kRound)), na, nb);   // fmaf(q, a_c, b_c)
    if constexpr (DT == SAND_BF16) {
      const __nv_bfloat162 v = __floats2bfloat162_rn(f2::lof(y), f2::hif(y));
      *reinterpret_cast<uint32_t*>(o) = *reinterpret_cast<const uint32_t*>(&v);
    } else {
      *reinterpret_cast<uint2*>(o) = make_uint2(f2::lo(y), f2::hi(y));
    }
  }
}
template <int DT>
constexpr int dt_bytes() { return DT == SAND_U8 ? 1 : (DT == SAND_BF16 ? 2 : 4); }

__device__ __forceinline__ float2 rint2(float2 v) {
  return __fadd2_rn(__fadd2_rn(v, make_float2(rs::kRound, rs::kRound)), make_float2(-rs::kRound, -rs::kRound));
}

// floor of a packed pair: s + 1.5*2^23 rounded toward -inf is 1.5*2^23 + floor(s) exactly for
// |s| < 2^22 (FADD2.RM), so the integer sits in the low mantissa bits
__device__ __forceinline__ uint64_t add_rm2(uint64_t a, uint64_t b) {
  uint64_t d;
  asm("add.rm.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}

#ifndef SAND_ROT_UNROLL
#define SAND_ROT_UNROLL 2
#endif
constexpr int kRotUnroll = SAND_ROT_UNROLL;   // rotation pixel-loop unroll (ILP for the tap loads)
#ifndef SAND_ROT_RPW
#define SAND_ROT_RPW 2
#endif
constexpr int kRotRPW = SAND_ROT_RPW;   // Q3 rows per warp per ring band (fewer barriers)

// Rotation (R#15) of all three Q2 planes in place. Q3 rows are computed band by band (one
// row per warp) into a ring of ring_rows (a power of two) rows, and row r is written back over
// Q2 row r once no later Q3 row can tap it: every tap of Q3 row y lies in Q2 rows
// [y - D, y + D]. Coordinates and fractions are computed once per pixel for the three channels.
__device__ __forceinline__ void rotate_inplace(const GroupParams& g, uint32_t q2, size_t plane, uint32_t ring,
                                               int ring_rows, int D, int Wo, int Ho, int warp, int nwarps,
                                               int lane) {
  using namespace rs;
  const float rc = g.rot_c, rsn = g.rot_s, nrs = -g.rot_s;
  const float cxo = (float)(Wo - 1) * 0.5f, cyo = (float)(Ho - 1) * 0.5f;
  const uint32_t P = (uint32_t)plane, rplane = (uint32_t)(ring_rows * Wo), rmask = (uint32_t)ring_rows - 1u;
  const uint64_t c2 = f2::pack(cxo, cyo), kr2 = f2::splat(kRound), nkr2 = f2::splat(-kRound);
  const uint64_t nb2 = f2::splat(-kBias), m1 = f2::splat(-1.f);
  int committed = 0;   // Q2 rows [0, committed) hold Q3 already
  for (int yb = 0; yb < Ho; yb += kRotRPW * nwarps) {
#pragma unroll 1
   for (int qr = 0; qr < kRotRPW; ++qr) {
    const int oy = yb + qr * nwarps + warp;
    if (oy < Ho) {
      const float yc = __fsub_rn((float)oy, cyo);
      const uint64_t txy = f2::pack(__fmul_rn(nrs, yc), __fmul_rn(rc, yc));   // row terms
      const uint32_t orow = ring + ((uint32_t)oy & rmask) * (uint32_t)Wo;
      float xc = __fsub_rn((float)lane, cxo);
      #pragma unroll (kRotUnroll)
      for (int ox = lane; ox < Wo; ox += 32, xc = __fadd_rn(xc, 32.f)) {
        // (sx, sy) = ((c*xc + (-s)*yc) + cx, (s*xc + c*yc) + cy), every op rounded (.rn ops
        // are not contracted)
        const uint64_t s2 = f2::add(f2::add(f2::pack(__fmul_rn(rc, xc), __fmul_rn(rsn, xc)), txy), c2);
        const uint64_t t = add_rm2(s2, kr2);                      // 1.5*2^23 + floor
        const uint64_t l = f2::fma(f2::add(t, nkr2), m1, s2);     // s - floor(s), exact
        const int x0 = (int)(f2::lo(t) - 0x4B400000u), y0 = (int)(f2::hi(t) - 0x4B400000u);
        const uint64_t lx = f2::splat(f2::lof(l));
        const float ly = f2::hif(l);
        const uint32_t a0 = q2 + (uint32_t)(y0 * Wo + x0);
        auto lerp = [&](uint32_t b00, uint32_t b01, uint32_t b10, uint32_t b11) {
          // rows packed: (t00, t10) and (t01, t11) as biased floats 2^23 + t
          const uint64_t T0 = f2::pack(0x4B000000u | b00, 0x4B000000u | b10);
          const uint64_t T1 = f2::pack(0x4B000000u | b01, 0x4B000000u | b11);
          const uint64_t h = f2::fma(lx, f2::fma(T0, m1, T1), f2::add(T0, nb2));   // (h0, h1)
          const float h0 = f2::lof(h), h1 = f2::hif(h);
          return __float_as_uint(__fadd_rn(__fmaf_rn(ly, __fsub_rn(h1, h0), h0), kRound));   // rint -> low byte
        };
        if ((unsigned)x0 < (unsigned)(Wo - 1) && (unsigned)y0 < (unsigned)(Ho - 1)) {
#pragma unroll
          for (int c = 0; c < 3; ++c) {
            const uint32_t a = a0 + (uint32_t)c * P, aw = a + (uint32_t)Wo;
            stsu8(orow + (uint32_t)c * rplane + (uint32_t)ox, lerp(ldsu8(a), ldsu8(a + 1), ldsu8(aw), ldsu8(aw + 1)));
          }
        } else {                                 // taps outside the image read 0 (fill=None)
          const bool in00 = x0 >= 0 && x0 < Wo && y0 >= 0 && y0 < Ho, in01 = x0 + 1 >= 0 && x0 + 1 < Wo && y0 >= 0 && y0 < Ho;
          const bool in10 = x0 >= 0 && x0 < Wo && y0 + 1 >= 0 && y0 + 1 < Ho;
          const bool in11 = x0 + 1 >= 0 && x0 + 1 < Wo && y0 + 1 >= 0 && y0 + 1 < Ho;
#pragma unroll
          for (int c = 0; c < 3; ++c) {
            const uint32_t a = a0 + (uint32_t)c * P;
            stsu8(orow + (uint32_t)c * rplane + (uint32_t)ox,
                  lerp(in00 ? ldsu8(a) : 0u, in01 ? ldsu8(a + 1) : 0u, in10 ? ldsu8(a + (uint32_t)Wo) : 0u,
                       in11 ? ldsu8(a + (uint32_t)Wo + 1) : 0u));
          }
        }
      }
    }
   }
    __syncthreads();                     // ring rows of this band written; Q2 reads done
    const int last = min(yb + kRotRPW * nwarps, Ho) - 1;
    const int upto = last + 1 >= Ho ? Ho : max(committed, last - D + 1);   // rows < upto are dead in Q2
    if (upto > committed) {              // write back Q3 rows [committed, upto) of the three planes
#pragma unroll 1
      for (int c = 0; c < 3; ++c) {
        for (int row = committed + warp; row < upto; row += nwarps) {
          const uint32_t from = ring + (uint32_t)c * rplane + ((uint32_t)row & rmask) * (uint32_t)Wo;
          const uint32_t to = q2 + (uint32_t)c * P + (uint32_t)(row * Wo);
          if ((Wo & 3) == 0) {
            for (int x = 4 * lane; x < Wo; x += 128) sts32(to + (uint32_t)x, st::lds32(from + (uint32_t)x));
          } else {
            for (int x = lane; x < Wo; x += 32) stsu8(to + (uint32_t)x, ldsu8(from + (uint32_t)x));
          }
        }
      }
      committed = upto;
    }
    __syncthreads();
  }
}

// Rotation (R#15) of the three Q2 planes straight to the output when no blur follows: Q3 is
// rint'ed, normalised (R#17) and stored per pixel (2/4/1-byte stores, a warp writes one
// contiguous row segment per channel). Q2 is only read, so no barriers are needed.
template <int DT>
__device__ __forceinline__ void rotate_direct(const GroupParams& g, uint32_t q2, size_t plane, int Wo, int Ho,
                                              int warp, int nwarps, int lane, uint8_t* const (&obase)[3],
                                              const float (&na)[3], const float (&nb)[3]) {
  using namespace rs;
  const float rc = g.rot_c, rsn = g.rot_s, nrs = -g.rot_s;
  const float cxo = (float)(Wo - 1) * 0.5f, cyo = (float)(Ho - 1) * 0.5f;
  const uint32_t P = (uint32_t)plane;
  const uint64_t c2 = f2::pack(cxo, cyo), kr2 = f2::splat(kRound), nkr2 = f2::splat(-kRound);
  const uint64_t nb2 = f2::splat(-kBias), m1 = f2::splat(-1.f);
  for (int oy = warp; oy < Ho; oy += nwarps) {
    const float yc = __fsub_rn((float)oy, cyo);
    const uint64_t txy = f2::pack(__fmul_rn(nrs, yc), __fmul_rn(rc, yc));
    uint8_t* op[3];                      // this lane's output pixel of the row, per channel
#pragma unroll
    for (int c = 0; c < 3; ++c) op[c] = obase[c] + ((size_t)oy * Wo + lane) * dt_bytes<DT>();
    float xc = __fsub_rn((float)lane, cxo);
    #pragma unroll (kRotUnroll)
    for (int ox = lane; ox < Wo;
         ox += 32, xc = __fadd_rn(xc, 32.f), op[0] += 32 * dt_bytes<DT>(), op[1] += 32 * dt_bytes<DT>(),
         op[2] += 32 * dt_bytes<DT>()) {
      const uint64_t s2 = f2::add(f2::add(f2::pack(__fmul_rn(rc, xc), __fmul_rn(rsn, xc)), txy), c2);
      const uint64_t t = add_rm2(s2, kr2);
      const uint64_t l = f2::fma(f2::add(t, nkr2), m1, s2);
      const int x0 = (int)(f2::lo(t) - 0x4B400000u), y0 = (int)(f2::hi(t) - 0x4B400000u);
      const uint64_t lx = f2::splat(f2::lof(l));
      const float ly = f2::hif(l);
      const uint32_t a0 = q2 + (uint32_t)(y0 * Wo + x0);
      auto emit = [&](int c, uint32_t b00, uint32_t b01, uint32_t b10, uint32_t b11) {
        const uint64_t T0 = f2::pack(0x4B000000u | b00, 0x4B000000u | b10);
        const uint64_t T1 = f2::pack(0x4B000000u | b01, 0x4B000000u | b11);
        const uint64_t h = f2::fma(lx, f2::fma(T0, m1, T1), f2::add(T0, nb2));
        const float h0 = f2::lof(h), h1 = f2::hif(h);
        const float tq = __fadd_rn(__fmaf_rn(ly, __fsub_rn(h1, h0), h0), kRound);   // 1.5*2^23 + q
        uint8_t* o = op[c];
        if constexpr (DT == SAND_U8) {
          *o = (uint8_t)(__float_as_uint(tq) & 0xffu);
        } else {
          const float y = __fmaf_rn(__fadd_rn(tq, -kRound), na[c], nb[c]);
          if constexpr (DT == SAND_BF16) *reinterpret_cast<__nv_bfloat16*>(o) = __float2bfloat16_rn(y);
          else *reinterpret_cast<float*>(o) = y;
        }
      };
      if ((unsigned)x0 < (unsigned)(Wo - 1) && (unsigned)y0 < (unsigned)(Ho - 1)) {
#pragma unroll
        for (int c = 0; c < 3; ++c) {
          const uint32_t a = a0 + (uint32_t)c * P, aw = a + (uint32_t)Wo;
          emit(c, ldsu8(a), ldsu8(a + 1), ldsu8(aw), ldsu8(aw + 1));
        }
      } else {                                   // taps outside the image read 0 (fill=None)
        const bool in00 = x0 >= 0 && x0 < Wo && y0 >= 0 && y0 < Ho, in01 = x0 + 1 >= 0 && x0 + 1 < Wo && y0 >= 0 && y0 < Ho;
        const bool in10 = x0 >= 0 && x0 < Wo && y0 + 1 >= 0 && y0 + 1 < Ho;
        const bool in11 = x0 + 1 >= 0 && x0 + 1 < Wo && y0 + 1 >= 0 && y0 + 1 < Ho;
#pragma unroll
        for (int c = 0; c < 3; ++c) {
          const uint32_t a = a0 + (uint32_t)c * P;
          emit(c, in00 ? ldsu8(a) : 0u, in01 ? ldsu8(a + 1) : 0u, in10 ? ldsu8(a + (uint32_t)Wo) : 0u,
               in11 ? ldsu8(a + (uint32_t)Wo + 1) : 0u);
        }
      }
    }
  }
}

#ifndef SAND_BLUR_BX
#define SAND_BLUR_BX 8
#endif
#ifndef SAND_BLUR_BV
#define SAND_BLUR_BV 16
#endif
constexpr int kBX = SAND_BLUR_BX;   // blur: columns per thread in the horizontal pass (multiple of 4)
constexpr int kBV = SAND_BLUR_BV;   // blur: rows per thread in the vertical pass

// Byte (relative to the window's 4-aligned word base) of horizontal window element k, i.e. of
// column x0 - R + k reflected (R#16), for the three block kinds: MODE 0 interior (base
// x0 - R - kOff), MODE 1 left border (x0 = 0, base 0), MODE 2 right border (x0 = Wo - kBX,
// base x0 - R - kOff). All compile-time for a given (R, MODE).
template <int R>
constexpr int blur_koff() { return (4 - (R & 3)) & 3; }
template <int R, int MODE>
__host__ __device__ constexpr int widx(int k) {
  return MODE == 0 ? blur_koff<R>() + k
                   : (MODE == 1 ? (k < R ? R - k : k - R)
                                : (k < kBX + R ? blur_koff<R>() + k : blur_koff<R>() + 2 * (kBX - 1) + 2 * R - k));
}
template <int R, int MODE>
constexpr int wwords() {
  return (MODE == 0 ? blur_koff<R>() + kBX + 2 * R - 1 : (MODE == 1 ? kBX + R - 1 : blur_koff<R>() + kBX + R - 1)) / 4 + 1;
}

// horizontal pass of one block: kBX outputs of strip rows (a, b) packed as pairs; window element
// k feeds outputs o = k - i (taps i in order 0..2R, R#16), one converted element live at a time
template <int R, int MODE>
__device__ __forceinline__ void hblur_block(uint32_t rowa, uint32_t rowb, uint32_t wb, const float (&wt)[2 * R + 1],
                                            uint64_t (&accs)[kBX]) {
  constexpr int kW = wwords<R, MODE>();
  uint32_t wa[kW], wv[kW];
#pragma unroll
  for (int k = 0; k < kW; ++k) {
    wa[k] = st::lds32(rowa + wb + 4u * k);
    wv[k] = st::lds32(rowb + wb + 4u * k);
  }
#pragma unroll
  for (int o = 0; o < kBX; ++o) accs[o] = 0ull;
#pragma unroll
  for (int k = 0; k < kBX + 2 * R; ++k) {
    const int bi = widx<R, MODE>(k);
    // biased floats 2^23 + byte of both rows, then one packed subtract
    const uint32_t fa = __byte_perm(wa[bi >> 2], 0x4B000000u, 0x7440 | (bi & 3));
    const uint32_t fb = __byte_perm(wv[bi >> 2], 0x4B000000u, 0x7440 | (bi & 3));
    const uint64_t v = rs::f2::add(rs::f2::pack(fa, fb), rs::f2::splat(-rs::kBias));
#pragma unroll
    for (int o = 0; o < kBX; ++o)
      if (k - o >= 0 && k - o <= 2 * R) accs[o] = rs::f2::fma(rs::f2::splat(wt[k - o]), v, accs[o]);
  }
}

// Separable Gaussian blur of one channel plane with radius R (R#16): horizontal pass into the
// fp32 scratch in row strips, vertical pass, rint (Q4), normalise and store. Every output's taps
// are accumulated from 0 in order i = 0..2R with fmaf in both passes (bit-identical to the
// oracle). Fast path (R <= kBX, Wo % kBX == 0, Wo % 4 == 0, Wo >= 2 kBX + R + 3): word loads with
// compile-time reflect maps for the border blocks; otherwise per-byte loads with reflect.
template <int DT, bool VEC, int R>
__device__ __forceinline__ void blur_plane(const LaunchParams& p, const GroupParams& g, const ChDests& cd,
                                           uint32_t src, uint32_t scratch, size_t scratch_bytes, int Wo, int Ho,
                                           int tid, int nthr) {
  const int pairs = (Wo + 1) >> 1;
  const int cap_rows = (int)(scratch_bytes / ((size_t)Wo * 4));   // fp32 rows the scratch holds
  // vertical mapping: G groups of `pairs` threads, each group takes kBV-row blocks of the strip
  const int G = max(1, nthr / pairs);
  const int vgrp = tid / pairs, vpr = tid - vgrp * pairs;
  // strip height: the largest multiple of G * kBV that fits (so row blocks spread evenly over
  // the groups), else whatever fits
  int S = ((cap_rows - 2 * R) / (G * kBV)) * (G * kBV);
  if (S <= 0) S = cap_rows - 2 * R;
  S = min(S, Ho);
  float wt[2 * R + 1];
#pragma unroll
  for (int i = 0; i <= 2 * R; ++i) wt[i] = __ldg(&g.blur_w[i]);
  // the compile-time border maps cover the first and last block only, so every other block
  // must be interior: R <= kBX (R > kBX, i.e. sigma > 2.1 with kBX = 8, takes the generic path)
  const bool fast = R <= kBX && (Wo & 3) == 0 && Wo % kBX == 0 && Wo >= 2 * kBX + R + 3;
  const int xblocks = fast ? Wo / kBX : (Wo + kBX - 1) / kBX;
  constexpr int kOff = blur_koff<R>();
  for (int ys = 0; ys < Ho; ys += S) {
    const int ns = min(S, Ho - ys);
    const int jrows = ns + 2 * R;          // strip row j <-> image row reflect(ys - R + j)
    const int half = (jrows + 1) >> 1;
    // ---- horizontal pass: unit = (strip rows j, j + half) x block of kBX columns. Interior
    // units first (lanes along the row), then the two border blocks of every row pair, so a
    // warp runs one block kind.
    if (fast) {
      const int nib = xblocks - 2;         // interior blocks per row
      const int n_int = half * nib, n_all = half * xblocks;
      for (int e = tid; e < n_all; e += nthr) {
        int j, x0, mode;
        if (e < n_int) {
          j = e / nib;
          x0 = (e - j * nib + 1) * kBX;
          mode = 0;
        } else {
          const int e2 = e - n_int;
          j = e2 >> 1;
          mode = 1 + (e2 & 1);
          x0 = mode == 1 ? 0 : Wo - kBX;
        }
        const int ja2 = j, jb2 = min(j + half, jrows - 1);
        const uint32_t rowa = src + (uint32_t)(reflect(ys - R + ja2, Ho) * Wo);
        const uint32_t rowb = src + (uint32_t)(reflect(ys - R + jb2, Ho) * Wo);
        uint64_t accs[kBX];
        if (mode == 0) hblur_block<R, 0>(rowa, rowb, (uint32_t)(x0 - R - kOff), wt, accs);
        else if (mode == 1) hblur_block<R, 1>(rowa, rowb, 0u, wt, accs);
        else hblur_block<R, 2>(rowa, rowb, (uint32_t)(x0 - R - kOff), wt, accs);
#pragma unroll
        for (int o = 0; o < kBX; o += 4) {   // 16 B stores: 4 columns of one strip row
          st::sts128(scratch + 4u * (uint32_t)(ja2 * Wo + x0 + o),
                     make_uint4(rs::f2::lo(accs[o]), rs::f2::lo(accs[o + 1]), rs::f2::lo(accs[o + 2]),
                                rs::f2::lo(accs[o + 3])));
          st::sts128(scratch + 4u * (uint32_t)(jb2 * Wo + x0 + o),
                     make_uint4(rs::f2::hi(accs[o]), rs::f2::hi(accs[o + 1]), rs::f2::hi(accs[o + 2]),
                                rs::f2::hi(accs[o + 3])));
        }
      }
    } else {
      for (int e = tid; e < half * xblocks; e += nthr) {
        const int j = e / xblocks, x0 = (e - j * xblocks) * kBX;
        const int ja2 = j, jb2 = min(j + half, jrows - 1);
        const uint32_t rowa = src + (uint32_t)(reflect(ys - R + ja2, Ho) * Wo);
        const uint32_t rowb = src + (uint32_t)(reflect(ys - R + jb2, Ho) * Wo);
        uint64_t accs[kBX];
#pragma unroll
        for (int o = 0; o < kBX; ++o) accs[o] = 0ull;
#pragma unroll
        for (int k = 0; k < kBX + 2 * R; ++k) {
          const int xx = reflect(min(x0 - R + k, 2 * Wo - 2), Wo);
          const uint64_t v = rs::f2::pack(u8f(ldsu8(rowa + (uint32_t)xx)), u8f(ldsu8(rowb + (uint32_t)xx)));
#pragma unroll
          for (int o = 0; o < kBX; ++o)
            if (k - o >= 0 && k - o <= 2 * R) accs[o] = rs::f2::fma(rs::f2::splat(wt[k - o]), v, accs[o]);
        }
#pragma unroll
        for (int o = 0; o < kBX; ++o) {
          if (x0 + o < Wo) {
            sts32(scratch + 4u * (uint32_t)(ja2 * Wo + x0 + o), rs::f2::lo(accs[o]));
            sts32(scratch + 4u * (uint32_t)(jb2 * Wo + x0 + o), rs::f2::hi(accs[o]));
          }
        }
      }
    }
    __syncthreads();
    // ---- vertical pass: thread = column pair (x, x+1) x blocks of kBV output rows; window rows
    // feed the outputs in tap order as in the horizontal pass
    if (vgrp < G) {
      const int nblk = (ns + kBV - 1) / kBV;
      const int ox = 2 * vpr;
      const bool has_b = ox + 1 < Wo;
      const bool pair_ok = has_b && !(Wo & 1);
      const uint32_t rstep = 4u * (uint32_t)Wo;
      const bool fast_st = cd.nd == 1 && pair_ok;
      uint8_t* const obase = cd.d0.base;
      const uint64_t na = rs::f2::splat(cd.d0.a), nb = rs::f2::splat(cd.d0.b);
      for (int blk = vgrp; blk < nblk; blk += G) {
        const int y0 = blk * kBV;
        uint64_t accs[kBV];
#pragma unroll
        for (int o = 0; o < kBV; ++o) accs[o] = 0ull;
        const uint32_t a0 = scratch + 4u * (uint32_t)(y0 * Wo + ox);
        if (pair_ok && y0 + kBV + 2 * R <= jrows) {   // fast path: no per-row branches or clamps
#pragma unroll
          for (int k = 0; k < kBV + 2 * R; ++k) {
            const float2 f = lds64f(a0 + rstep * k);
            const uint64_t v = rs::f2::pack(f.x, f.y);
#pragma unroll
            for (int o = 0; o < kBV; ++o)
              if (k - o >= 0 && k - o <= 2 * R) accs[o] = rs::f2::fma(rs::f2::splat(wt[k - o]), v, accs[o]);
          }
        } else {
#pragma unroll
          for (int k = 0; k < kBV + 2 * R; ++k) {
            // rows past the strip only feed outputs that are not stored: clamp their address
            const uint32_t a = scratch + 4u * (uint32_t)(min(y0 + k, jrows - 1) * Wo + ox);
            const uint32_t xa = st::lds32(a), xb = st::lds32(a + (has_b ? 4u : 0u));
            const uint64_t v = rs::f2::pack(xa, has_b ? xb : 0u);
#pragma unroll
            for (int o = 0; o < kBV; ++o)
              if (k - o >= 0 && k - o <= 2 * R) accs[o] = rs::f2::fma(rs::f2::splat(wt[k - o]), v, accs[o]);
          }
        }
        if constexpr (DT >= 0) {
          if (fast_st) {                     // one destination: incremental row pointer
            uint8_t* o = obase + ((size_t)(ys + y0) * Wo + ox) * dt_bytes<DT>();
            const uint32_t rsb = (uint32_t)Wo * dt_bytes<DT>();
            if (y0 + kBV <= ns) {            // whole block: no per-row checks
#pragma unroll
              for (int oo = 0; oo < kBV; ++oo)
                put_pair<DT>(o + oo * rsb, rs::f2::add(accs[oo], rs::f2::splat(rs::kRound)), na, nb);
            } else {
#pragma unroll
              for (int oo = 0; oo < kBV; ++oo) {
                if (y0 + oo >= ns) break;
                put_pair<DT>(o + oo * rsb, rs::f2::add(accs[oo], rs::f2::splat(rs::kRound)), na, nb);
              }
            }
            continue;
          }
        }
#pragma unroll
        for (int o = 0; o < kBV; ++o) {
          if (y0 + o >= ns) break;
          store_q<DT, VEC>(p, cd, ys + y0 + o, ox, Wo, rint2(make_float2(rs::f2::lof(accs[o]), rs::f2::hif(accs[o]))),
                           has_b);
        }
      }
    }
    __syncthreads();
  }
}

// Colour jitter (R#30) on the three Q2 planes in place, after flip, before rotation:
// the ops of the drawn order one after the other, each a full pass (barrier between), every fp32
// operation rounded on its own as in the oracle; contrast's mean is an exact integer sum of the
// floored greys (block reduction) divided once. s_acc: 4 free bytes of shared memory.
__device__ __forceinline__ float jit_gray(float r, float g, float b) {
  return floorf(__fadd_rn(__fadd_rn(__fmul_rn(r, 0.2989f), __fmul_rn(g, 0.587f)), __fmul_rn(b, 0.114f)));
}
__device__ __forceinline__ uint32_t jit_u8(float v) {   // clamp to [0, 255], truncate (torch float -> uint8)
  return __float2uint_rz(fminf(fmaxf(v, 0.f), 255.f));
}
__device__ void jitter_planes(const GroupParams& g, uint32_t q2, uint32_t plane, int n, uint32_t s_acc, int tid,
                              int nthr) {
  const int ord = g.jit_order;             // op of step s at bits 4 s (view.cpp)
  for (int step = 0; step < 3; ++step) {
    const int op = (ord >> (4 * step)) & 0xf;
    const float fx = g.jit_f[op], fa = g.jit_a[op];
    float mean = 0.f;
    if (op == 1) {                         // contrast: mean grey of the current image
      if (tid == 0) sts32(s_acc, 0u);
      __syncthreads();
      uint32_t sum = 0;
      for (int i = tid; i < n; i += nthr)
        sum += (uint32_t)jit_gray(u8f(ldsu8(q2 + i)), u8f(ldsu8(q2 + plane + i)), u8f(ldsu8(q2 + 2 * plane + i)));
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
      if ((tid & 31) == 0) asm volatile("red.shared.add.u32 [%0], %1;" ::"r"(s_acc), "r"(sum) : "memory");
      __syncthreads();
      mean = __fdiv_rn((float)st::lds32(s_acc), (float)n);
    }
    for (int i = tid; i < n; i += nthr) {
      const float r = u8f(ldsu8(q2 + i)), gg = u8f(ldsu8(q2 + plane + i)), b = u8f(ldsu8(q2 + 2 * plane + i));
      float o0, o1, o2;
      if (op == 0) {                       // brightness
        o0 = __fmul_rn(r, fx);
        o1 = __fmul_rn(gg, fx);
        o2 = __fmul_rn(b, fx);
      } else {                             // contrast (blend with the mean) or saturation (with the grey)
        const float other = __fmul_rn(op == 1 ? mean : jit_gray(r, gg, b), fa);
        o0 = __fadd_rn(__fmul_rn(r, fx), other);
        o1 = __fadd_rn(__fmul_rn(gg, fx), other);
        o2 = __fadd_rn(__fmul_rn(b, fx), other);
      }
      stsu8(q2 + i, jit_u8(o0));
      stsu8(q2 + plane + i, jit_u8(o1));
      stsu8(q2 + 2 * plane + i, jit_u8(o2));
    }
    __syncthreads();
  }
}

}  // namespace sc

template <int DT, bool VEC>
__global__ void __launch_bounds__(512, 1) k_stencil2(const LaunchParams p, sc::Shape sh, int maxWo) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  using namespace rs;
  using namespace sc;
  const WorkItem w = p.items[blockIdx.x];
  if (!(w.flags & 1u)) return;
  const GroupParams& g = p.groups[w.gp];
  const int Wo = g.out_w, Ho = g.out_h;
  const int tid = threadIdx.x, nthr = blockDim.x;
  const int warp = tid >> 5, lane = tid & 31, nwarps = nthr >> 5;
  uint32_t s_base = (uint32_t)__cvta_generic_to_shared(smem_raw);
  asm volatile("" : "+r"(s_base));
  const uint32_t q2 = s_base;                                  // 3 planes of sh.plane bytes
  const uint32_t ureg = s_base + (uint32_t)(3 * sh.plane);     // band buffers / Q3 plane
  uint2* ctab = reinterpret_cast<uint2*>(smem_raw + 3 * sh.plane);
  uint4* rtab = reinterpret_cast<uint4*>(smem_raw + 3 * sh.plane + a16((size_t)maxWo * 8));
  const uint32_t s_rtab = ureg + (uint32_t)a16((size_t)maxWo * 8);
  const uint32_t s_grid = ureg + (uint32_t)(a16((size_t)maxWo * 8) + a16((size_t)sh.R * 16));
  const uint32_t s_rawb = s_grid + (uint32_t)(sh.grid_rows * sh.gw * 4);
  const uint32_t* dests = p.dests + w.dest_begin;
  const int nd = (int)w.n_dest;

  // ------------------------------------------------------------- phase 1: Q2 planes
  const int x_lo = tap0(g.sc_x, g.off_x, 0, g.org_x);
  int x_hi, dmy;
  float fl;
  tap(g.sc_x, g.off_x, Wo - 1, g.lim_x, g.org_x, dmy, x_hi, fl);
  const int x16 = x_lo & ~15;
  const int gw = ((x_hi + 16) & ~15) - x16;
  const uint32_t rowbytes = (uint32_t)gw * 4u;
  const uint8_t* Yp = p.slab + w.y_off;
  const uint8_t* UVp = Yp + (size_t)w.pitch * w.src_h;
  // source rows of the band starting at output row oy_lo
  auto band = [&](int oy_lo, int& nr, int& y_lo, int& y_hi) {
    nr = min(sh.R, Ho - oy_lo);
    y_lo = tap0(g.sc_y, g.off_y, oy_lo, g.org_y);
    int d0;
    float f0;
    tap(g.sc_y, g.off_y, oy_lo + nr - 1, g.lim_y, g.org_y, d0, y_hi, f0);
  };
  {                                           // band 0's NV12 rows are in flight while the tables are built
    int nr0, ylo0, yhi0;
    band(0, nr0, ylo0, yhi0);
    st::stage_rows_cp(s_rawb, Yp + x16, UVp + x16, w.pitch, gw, ylo0, yhi0, warp, nwarps, lane);
  }
  for (int j = tid; j < Wo; j += nthr) {
    int x0, x1;
    float lx;
    tap(g.sc_x, g.off_x, j, g.lim_x, g.org_x, x0, x1, lx);
    ctab[j] = make_uint2((uint32_t)(x0 - x16) | ((uint32_t)(x1 - x16) << 16), __float_as_uint(lx));
  }
  const int pairs = (Wo + 1) >> 1;
  const int groups = max(1, nthr / pairs);
  const int grp = tid / pairs, pr = tid - grp * pairs;
  for (int oy_lo = 0; oy_lo < Ho; oy_lo += sh.R) {
    int nr, y_lo, y_hi;
    band(oy_lo, nr, y_lo, y_hi);
    asm volatile("cp.async.wait_group 0;\n" ::: "memory");
    __syncthreads();                          // raw of this band landed; the previous walk is done with grid/rtab
    st::convert_rows(s_grid, s_rawb, gw, y_lo, y_hi, y_lo, 1 << 30, 5u, warp, nwarps, lane, p.cm);   // no wrap
    for (int r = tid; r < nr; r += nthr) {
      int y0, y1;
      float ly;
      tap(g.sc_y, g.off_y, oy_lo + r, g.lim_y, g.org_y, y0, y1, ly);
      rtab[r] = make_uint4((uint32_t)(y0 - y_lo) * rowbytes, (uint32_t)(y1 - y_lo) * rowbytes, (uint32_t)y0,
                           __float_as_uint(ly));
    }
    __syncthreads();                          // grid + rtab ready, raw drained
    if (oy_lo + sh.R < Ho) {                  // the next band's rows load while this band is walked
      int nr1, ylo1, yhi1;
      band(oy_lo + sh.R, nr1, ylo1, yhi1);
      st::stage_rows_cp(s_rawb, Yp + x16, UVp + x16, w.pitch, gw, ylo1, yhi1, warp, nwarps, lane);
    }
    if (grp < groups && pr < pairs) {
      const int ox = 2 * pr;
      const bool has_b = ox + 1 < Wo;
      const bool even_w = !(Wo & 1);
      const int ja = g.flip ? Wo - 1 - ox : ox;
      const int jb = has_b ? (g.flip ? Wo - 2 - ox : ox + 1) : ja;
      const uint2 ta = ctab[ja], tb = ctab[jb];
      const uint32_t ca0 = 4u * (ta.x & 0xffffu), ca1 = 4u * (ta.x >> 16);
      const uint32_t cb0 = 4u * (tb.x & 0xffffu), cb1 = 4u * (tb.x >> 16);
      const uint64_t lx = f2::pack(ta.y, tb.y);
      const int per = (nr + groups - 1) / groups;
      const int r_lo = grp * per, r_hi = min(nr, r_lo + per);
      int have0 = -1, have1 = -1;
      Row3 S0, S1;
      for (int rr = r_lo; rr < r_hi; ++rr) {
        const uint4 rt = st::lds128(s_rtab + 16u * rr);
        const uint32_t o0 = s_grid + rt.x, o1 = s_grid + rt.y;
        const int y0 = (int)rt.z;
        const uint64_t ly = f2::splat(__uint_as_float(rt.w));
        const uint32_t pix = (uint32_t)((oy_lo + rr) * Wo + ox);
        auto put3 = [&](const Row3& top, const Row3& bot) {   // vertical lerp + rint -> Q2 planes
#pragma unroll
          for (int c = 0; c < 3; ++c) {
            const uint64_t dv = f2::fma(top.h[c], f2::splat(-1.f), bot.h[c]);
            const uint64_t tq = rint_biased(f2::fma(ly, dv, top.h[c]));   // low bytes = q
            const uint32_t pair = __byte_perm(f2::lo(tq), f2::hi(tq), 0x0040);
            const uint32_t plane = q2 + (uint32_t)(c * sh.plane) + pix;
            if (VEC || (has_b && even_w)) {    // VEC: every width is even (host-checked)
              if (VEC || has_b) stsu16(plane, pair);   // pix is even: 2-byte aligned
              else stsu8(plane, pair);
            } else {                           // odd plane width: pixel pairs can straddle
              stsu8(plane, pair);
              if (has_b) stsu8(plane + 1, pair >> 8);
            }
          }
        };
        if (y0 & 1) {
          if (have1 != y0) { st::hrow_s(S1, o0, ca0, ca1, cb0, cb1, lx); have1 = y0; }
          if (o1 != o0) {
            if (have0 != y0 + 1) { st::hrow_s(S0, o1, ca0, ca1, cb0, cb1, lx); have0 = y0 + 1; }
            put3(S1, S0);
          } else {
            put3(S1, S1);
          }
        } else {
          if (have0 != y0) { st::hrow_s(S0, o0, ca0, ca1, cb0, cb1, lx); have0 = y0; }
          if (o1 != o0) {
            if (have1 != y0 + 1) { st::hrow_s(S1, o1, ca0, ca1, cb0, cb1, lx); have1 = y0 + 1; }
            put3(S0, S1);
          } else {
            put3(S0, S0);
          }
        }
      }
    }
  }
  __syncthreads();

  // ------------------------------------------------------------- phase 1b: colour jitter (R#30)
  if (g.jit_on) jitter_planes(g, q2, (uint32_t)sh.plane, Wo * Ho, ureg, tid, nthr);

  // ------------------------------------------------------------- phase 2: per channel
  const int r = g.blur_on ? g.blur_r : 0;
  const float cxo = (float)(Wo - 1) * 0.5f, cyo = (float)(Ho - 1) * 0.5f;
  if constexpr (DT >= 0) {
    if (g.rot_on && !g.blur_on && nd == 1) {   // a8 + a10 straight to the output
      uint8_t* ob[3];
      float na[3], nb[3];
#pragma unroll
      for (int c = 0; c < 3; ++c) {
        const ChDest d = ch_dest(p, dests[0], c);
        ob[c] = d.base;
        na[c] = d.a;
        nb[c] = d.b;
      }
      rotate_direct<DT>(g, q2, sh.plane, Wo, Ho, warp, nwarps, lane, ob, na, nb);
      return;
    }
  }
  // a8 in place for all three channels when its ring fits the band/Q3 region; else per channel
  bool rotated = false;
  if (g.rot_on) {
    const float bound = fabsf(g.rot_s) * cxo + (1.f - g.rot_c) * cyo;
    const int D = (int)ceilf(bound) + 2;
    int ring_rows = 1;
    while (ring_rows < D + kRotRPW * nwarps + 1) ring_rows <<= 1;
    if ((size_t)ring_rows * 3 * Wo <= sh.ubytes && D < Ho) {
      rotate_inplace(g, q2, sh.plane, ureg, ring_rows, D, Wo, Ho, warp, nwarps, lane);
      rotated = true;
    }
  }
  // channels last to first: once channel c is done its plane joins the scratch of the next
  // (planes are contiguous and the band/Q3 region follows plane 2)
  for (int c = 2; c >= 0; --c) {
    ChDests cd;
    cd.nd = nd;
    cd.dests = dests;
    cd.c = c;
    cd.d0 = ch_dest(p, dests[0], c);
    if (nd > 1) cd.d1 = ch_dest(p, dests[1], c);
    uint32_t src = q2 + (uint32_t)(c * sh.plane);
    uint32_t scratch = q2 + (uint32_t)((c + 1) * sh.plane);
    size_t scratch_bytes = (size_t)(2 - c) * sh.plane + sh.ubytes;
    if (g.rot_on && !rotated) {              // a8: Q3 = rotate(Q2) (R#15), one channel
      const uint32_t q3 = ureg;
      const float rc = g.rot_c, rsn = g.rot_s, nrs = -g.rot_s;
      for (int oy = warp; oy < Ho; oy += nwarps) {
        const float yc = __fsub_rn((float)oy, cyo);
        const float tx = __fmul_rn(nrs, yc), ty = __fmul_rn(rc, yc);   // row terms of R#15
        const uint32_t orow = q3 + (uint32_t)(oy * Wo);
        float xc = __fsub_rn((float)lane, cxo);
        for (int ox = lane; ox < Wo; ox += 32, xc = __fadd_rn(xc, 32.f)) {
          // sx = (c*xc + (-s)*yc) + cx, sy = (s*xc + c*yc) + cy, every op rounded (scalar IEEE)
          const float sx = __fadd_rn(__fadd_rn(__fmul_rn(rc, xc), tx), cxo);
          const float sy = __fadd_rn(__fadd_rn(__fmul_rn(rsn, xc), ty), cyo);
          const float fx = floorf(sx), fy = floorf(sy);
          const float lxr = __fsub_rn(sx, fx), lyr = __fsub_rn(sy, fy);
          const int x0 = (int)fx, y0 = (int)fy;
          float t00, t01, t10, t11;
          if ((unsigned)x0 < (unsigned)(Wo - 1) && (unsigned)y0 < (unsigned)(Ho - 1)) {
            const uint32_t a0 = src + (uint32_t)(y0 * Wo + x0);
            t00 = u8f(ldsu8(a0));
            t01 = u8f(ldsu8(a0 + 1));
            t10 = u8f(ldsu8(a0 + (uint32_t)Wo));
            t11 = u8f(ldsu8(a0 + (uint32_t)Wo + 1));
          } else {                               // taps outside the image read 0 (fill=None)
            auto tapv = [&](int xx, int yy) {
              return (xx >= 0 && xx < Wo && yy >= 0 && yy < Ho) ? u8f(ldsu8(src + (uint32_t)(yy * Wo + xx))) : 0.f;
            };
            t00 = tapv(x0, y0);
            t01 = tapv(x0 + 1, y0);
            t10 = tapv(x0, y0 + 1);
            t11 = tapv(x0 + 1, y0 + 1);
          }
          const float h0 = __fmaf_rn(lxr, __fsub_rn(t01, t00), t00);
          const float h1 = __fmaf_rn(lxr, __fsub_rn(t11, t10), t10);
          // rint via +1.5*2^23: the integer lands in the low mantissa bits (0..255)
          const float tq = __fadd_rn(__fmaf_rn(lyr, __fsub_rn(h1, h0), h0), rs::kRound);
          stsu8(orow + (uint32_t)ox, __float_as_uint(tq) & 0xffu);
        }
      }
      __syncthreads();
      src = q3;
      scratch = q2 + (uint32_t)(c * sh.plane);   // this channel's Q2 plane (and the done ones) are free now
      scratch_bytes = (size_t)(3 - c) * sh.plane;
    }
    if (g.blur_on) {         // a9: separable Gaussian in strips (R#16)
      switch (r) {
        case 0: blur_plane<DT, VEC, 0>(p, g, cd, src, scratch, scratch_bytes, Wo, Ho, tid, nthr); break;
        case 1: blur_plane<DT, VEC, 1>(p, g, cd, src, scratch, scratch_bytes, Wo, Ho, tid, nthr); break;
        case 2: blur_plane<DT, VEC, 2>(p, g, cd, src, scratch, scratch_bytes, Wo, Ho, tid, nthr); break;
        case 3: blur_plane<DT, VEC, 3>(p, g, cd, src, scratch, scratch_bytes, Wo, Ho, tid, nthr); break;
        case 4: blur_plane<DT, VEC, 4>(p, g, cd, src, scratch, scratch_bytes, Wo, Ho, tid, nthr); break;
        case 5: blur_plane<DT, VEC, 5>(p, g, cd, src, scratch, scratch_bytes, Wo, Ho, tid, nthr); break;
        case 6: blur_plane<DT, VEC, 6>(p, g, cd, src, scratch, scratch_bytes, Wo, Ho, tid, nthr); break;
        case 7: blur_plane<DT, VEC, 7>(p, g, cd, src, scratch, scratch_bytes, Wo, Ho, tid, nthr); break;
        case 8: blur_plane<DT, VEC, 8>(p, g, cd, src, scratch, scratch_bytes, Wo, Ho, tid, nthr); break;
        case 9: blur_plane<DT, VEC, 9>(p, g, cd, src, scratch, scratch_bytes, Wo, Ho, tid, nthr); break;
        case 10: blur_plane<DT, VEC, 10>(p, g, cd, src, scratch, scratch_bytes, Wo, Ho, tid, nthr); break;
        default: blur_plane<DT, VEC, 11>(p, g, cd, src, scratch, scratch_bytes, Wo, Ho, tid, nthr); break;
      }
    } else {                                   // no blur: normalise + store the (rotated) plane
      if ((Wo & 3) == 0) {                     // 4 pixels per thread from one word
        const int q4 = Wo >> 2;
        const int dy = nthr / q4, dq = nthr - dy * q4;   // unit e = oy * q4 + q, stepped without divisions
        int oy = tid / q4, q = tid - oy * q4;
        for (; oy < Ho; oy += dy, q += dq, (q >= q4 ? (q -= q4, ++oy) : 0)) {
          const int ox = 4 * q;
          const uint32_t wv = st::lds32(src + (uint32_t)(oy * Wo + ox));
          // 1.5*2^23 + q per byte (the rint-result form put_pair takes)
          const uint64_t t01 = rs::f2::pack(__byte_perm(wv, 0x4B400000u, 0x7640), __byte_perm(wv, 0x4B400000u, 0x7641));
          const uint64_t t23 = rs::f2::pack(__byte_perm(wv, 0x4B400000u, 0x7642), __byte_perm(wv, 0x4B400000u, 0x7643));
          if constexpr (DT >= 0) {
            if (nd == 1) {
              const uint64_t na = rs::f2::splat(cd.d0.a), nb = rs::f2::splat(cd.d0.b);
              uint8_t* o = cd.d0.base + ((size_t)oy * Wo + ox) * dt_bytes<DT>();
              put_pair<DT>(o, t01, na, nb);
              put_pair<DT>(o + 2 * dt_bytes<DT>(), t23, na, nb);
              continue;
            }
          }
          const uint64_t q01 = rs::f2::add(t01, rs::f2::splat(-rs::kRound)), q23 = rs::f2::add(t23, rs::f2::splat(-rs::kRound));
          store_q<DT, VEC>(p, cd, oy, ox, Wo, make_float2(rs::f2::lof(q01), rs::f2::hif(q01)), true);
          store_q<DT, VEC>(p, cd, oy, ox + 2, Wo, make_float2(rs::f2::lof(q23), rs::f2::hif(q23)), true);
        }
      } else {
        for (int oy = warp; oy < Ho; oy += nwarps) {
          const uint32_t row = src + (uint32_t)(oy * Wo);
          for (int ox = 2 * lane; ox < Wo; ox += 64) {
            const bool has_b = ox + 1 < Wo;
            const float2 q = make_float2(u8f(ldsu8(row + ox)), has_b ? u8f(ldsu8(row + ox + 1)) : 0.f);
            store_q<DT, VEC>(p, cd, oy, ox, Wo, q, has_b);
          }
        }
      }
      __syncthreads();
    }
  }
}

}  // namespace sand
