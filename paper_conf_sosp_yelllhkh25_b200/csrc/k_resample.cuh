// k_resample.cuh — shared device helpers of the resample kernels (k_plain, k_stream, k_direct,
// k_copy, k_stencil2): the R#12 tap rule, packed fp32
// pair arithmetic (sm_100a FFMA2/FADD2), horizontal lerps of RGBx words, destinations and the
// vertical lerp / rint / normalise / store sequence (R#12, R#17). Every fp32 operation is the
// oracle's op sequence with IEEE rounding (byte->float via the 2^23 exponent trick and rint via
// +1.5*2^23 are exact for values in [0, 256)), so results are bit-identical to the oracle.
#pragma once

namespace sand {
namespace rs {

constexpr int kInlineDests = 2;            // destinations kept in registers
constexpr float kBias = 8388608.0f;        // 2^23
constexpr float kRound = 12582912.0f;      // 1.5 * 2^23

__host__ __device__ inline size_t a16(size_t x) { return (x + 15) & ~size_t(15); }

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

__device__ __forceinline__ Dest make_dest(const LaunchParams& p, uint32_t dest, int oy, int ox, bool fold = false) {
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
    d.b[c] = fold ? vc.bf[c] : vc.b[c];
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

}  // namespace rs

}  // namespace sand
