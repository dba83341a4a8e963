// k_stream.cuh — streaming resample kernel for mild scaling (source step <= 2 rows/cols per
// output row/col: Kinetics RRC, SlowFast short-side crops).
//
// One CTA = one work item (clip slot, source frame, group) x one super-band of SB output
// rows, processed as sub-bands of S rows:
//   * the NV12 rows a sub-band adds are copied HBM -> shared memory with cp.async one
//     sub-band ahead (double-buffered raw staging, all 16 B requests in flight; a4);
//   * they are converted once to RGBx words in a shared-memory ring of source rows; a
//     thread takes one UV word (two chroma samples) and the 2x4 luma pixels sharing it,
//     with the clamp folded into DPX add-max (VIADDMNMX) and bytes packed by PRMT (a5, Q1);
//   * each thread owns an output column pair for the whole super-band and keeps the
//     horizontal lerps of the current two source rows in registers across sub-bands (a6),
//     mirrored for flip (a7); vertical lerp, rint, normalise and the 4-byte stores to every
//     destination view follow (a10, a11).
// Shared memory is addressed with 32-bit shared-window addresses (ld/st.shared) so the hot
// loops carry no generic-address arithmetic. Per-CTA setup is amortised over SB rows and
// no source row is converted twice inside a super-band. Arithmetic is the R#11/R#12/R#17
// op sequence with IEEE rounding at each step: bit-identical to the oracle.
#pragma once

namespace sand {
namespace st {

using rs::a16;

struct Shape {      // host-chosen launch shape
  int SB;           // output rows per CTA
  int nsb;          // super-bands per item (ceil(maxHo / SB))
  int S;            // output rows per sub-band
  int ring;         // ring capacity in source rows (>= rows one sub-band spans)
  int raw_rows;     // raw staging capacity in rows (Y + UV)
  int gw;           // max row width in bytes of Y (= words of RGBx), multiple of 16
  uint32_t ring_magic;   // floor(2^32 / ring) + 1: x / ring == umulhi(x, ring_magic) for x < 2^16
  int opts;         // bit0: warp-row conversion units instead of flattened units (A/B switch)
};

__device__ __forceinline__ uint32_t ring_mod(uint32_t x, uint32_t ring, uint32_t magic) {
  return x - __umulhi(x, magic) * ring;
}
__device__ __forceinline__ uint32_t ring_mod(uint32_t x, const Shape& s) {
  return ring_mod(x, (uint32_t)s.ring, s.ring_magic);
}

__host__ __device__ inline size_t smem_bytes(const Shape& s, int maxWo) {
  return a16((size_t)maxWo * 8) + a16((size_t)s.SB * 16) + (size_t)s.ring * s.gw * 4 +
         a16((size_t)s.raw_rows * s.gw) + 16;   // + the staging mbarrier
}

__device__ __forceinline__ uint32_t lds32(uint32_t a) {
  uint32_t v;
  asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
  return v;
}
__device__ __forceinline__ uint4 lds128(uint32_t a) {
  uint4 v;
  asm volatile("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
  return v;
}
__device__ __forceinline__ void sts128(uint32_t a, uint4 v) {
  asm volatile("st.shared.v4.u32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w)
               : "memory");
}
__device__ __forceinline__ void cp_async16s(uint32_t s, const void* gmem) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s), "l"(gmem) : "memory");
}

// mbarrier / bulk-copy primitives (32-bit shared-window addresses)
__device__ __forceinline__ void mbar_init(uint32_t bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(bar), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint32_t bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n"
      "SAND_WAIT_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      " @!p bra SAND_WAIT_%=;\n}\n" ::"r"(bar),
      "r"(parity)
      : "memory");
}
// the same wait with a suspend-time hint: a warp whose data has not landed sleeps in the
// barrier instead of re-issuing try_wait (no issue slots taken from the SM's other warps)
__device__ __forceinline__ void mbar_wait_sleep(uint32_t bar, uint32_t parity) {
  asm volatile(
      "{\n .reg .pred p;\n"
      "SAND_WAITS_%=:\n"
      " mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1, %2;\n"
      " @!p bra SAND_WAITS_%=;\n}\n" ::"r"(bar),
      "r"(parity), "r"(1000000u)
      : "memory");
}
__device__ __forceinline__ void bulk_g2s(uint32_t dst, const void* src, uint32_t bytes, uint32_t bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(dst),
               "l"(src), "r"(bytes), "r"(bar)
               : "memory");
}

// Y rows [ya, yb] then UV rows [ya>>1, yb>>1] -> raw (shared address), gw bytes per row, as
// one bulk copy (TMA engine) per row issued by thread `row`; completion is counted in bytes
// on the buffer's mbarrier. y0/uv0: global addresses of column x16 of Y row 0 / UV row 0
// (16 B aligned: store rows are 64 B aligned, x16 is a multiple of 16, gw of 16).
__device__ __forceinline__ void stage_rows(uint32_t raw, uint32_t bar, const uint8_t* y0, const uint8_t* uv0,
                                           uint32_t pitch, int gw, int ya, int yb, int tid, int nthr) {
  const int ny = yb - ya + 1, u0 = ya >> 1, nuv = (yb >> 1) - u0 + 1;
  if (tid == 0) mbar_arrive_expect_tx(bar, (uint32_t)((ny + nuv) * gw));
  for (int r = tid; r < ny + nuv; r += nthr) {
    const uint8_t* src = r < ny ? y0 + (size_t)(ya + r) * pitch : uv0 + (size_t)(u0 + r - ny) * pitch;
    bulk_g2s(raw + (uint32_t)(r * gw), src, (uint32_t)gw, bar);
  }
}

// cp.async variant (k_stencil): warps take rows, lanes take 16 B chunks
__device__ __forceinline__ void stage_rows_cp(uint32_t raw, const uint8_t* y0, const uint8_t* uv0, uint32_t pitch,
                                              int gw, int ya, int yb, int warp, int nwarps, int lane) {
  const int ny = yb - ya + 1, u0 = ya >> 1, nuv = (yb >> 1) - u0 + 1;
  const int chunks = gw >> 4;
  for (int r = warp; r < ny + nuv; r += nwarps) {
    const uint8_t* src = r < ny ? y0 + (size_t)(ya + r) * pitch : uv0 + (size_t)(u0 + r - ny) * pitch;
    const uint32_t dst = raw + (uint32_t)(r * gw);
#pragma unroll 1
    for (int k = lane; k < chunks; k += 32) cp_async16s(dst + 16u * k, src + 16 * k);
  }
  asm volatile("cp.async.commit_group;\n" ::: "memory");
}

// chroma terms (R#11 / R#29, matrix m) of the sample whose U is at bit SHIFT of the UV word
struct Chroma3 {
  int r, g, b;
};
template <int SHIFT>
__device__ __forceinline__ Chroma3 chroma_at(uint32_t uv, const ColorM& m) {
  // raw bytes U, V (one PRMT each); the -128 offsets are folded into the IMAD addends:
  // vr (V - 128) = vr V + kr etc. (exact integer arithmetic)
  const int u = (int)__byte_perm(uv, 0u, 0x4440 | (SHIFT / 8));
  const int v = (int)__byte_perm(uv, 0u, 0x4440 | (SHIFT / 8 + 1));
  return {m.vr * v + m.kr, m.vg * v + (m.ug * u + m.kg), m.ub * u + m.kb};
}

// RGBx word of luma Y with chroma c: sat((yy + term) >> 20) per channel (OpenCV integer
// BT.601), computed as relu(min(yy + term, 2^28 - 1)) >> 4 (one DPX VIADDMNMX.RELU), whose
// byte 2 is the channel; PRMT gathers the three bytes and the exponent byte 0x4B tops the word
// (see rs::biased).
__device__ __forceinline__ uint32_t rgbx_dpx(uint32_t Y, const Chroma3& c, const ColorM& m) {
  const int yy = (int)max(Y, 16u) * m.cy + m.yk;
  // x >> 4 of the clamped sums as IMAD.HI (FMA pipe) to relieve the ALU pipe
  const uint32_t mr = __umulhi((uint32_t)__viaddmin_s32_relu(yy, c.r, 0x0FFFFFFF), 1u << 28);
  const uint32_t mg = __umulhi((uint32_t)__viaddmin_s32_relu(yy, c.g, 0x0FFFFFFF), 1u << 28);
  const uint32_t mb = __umulhi((uint32_t)__viaddmin_s32_relu(yy, c.b, 0x0FFFFFFF), 1u << 28) + 0x4B000000u;
  return __byte_perm(__byte_perm(mr, mg, 0x0062), mb, 0x7610);
}

// byte I of w, zero-extended (one PRMT)
template <int I>
__device__ __forceinline__ uint32_t byte_of(uint32_t w) {
  return __byte_perm(w, 0u, 0x4440 | I);
}

// convert staged rows [ya, yb] into the ring (slot = (y - y_first) % ring_rows)
__device__ __forceinline__ void convert_rows(uint32_t ring, uint32_t raw, int gw, int ya, int yb, int y_first,
                                             int ring_rows, uint32_t ring_magic, int warp, int nwarps, int lane,
                                             const ColorM& cm) {
  const int ny = yb - ya + 1;
  if (ny <= 0) return;
  const int u0 = ya >> 1, nuv = (yb >> 1) - u0 + 1;
  const uint32_t rawUV = raw + (uint32_t)(ny * gw);
  const int q4 = gw >> 2;                      // 4-pixel groups per row
  const uint32_t rowbytes = (uint32_t)gw * 4u;
  for (int u = warp; u < nuv; u += nwarps) {
    const int yt = 2 * (u0 + u);
    const bool top = yt >= ya, bot = yt + 1 <= yb;
    const int st = (int)ring_mod((uint32_t)(yt - y_first + ring_rows), (uint32_t)ring_rows, ring_magic);   // yt may be y_first - 1
    const int sb = st + 1 == ring_rows ? 0 : st + 1;
    const uint32_t yrow_t = raw + (uint32_t)((yt - ya) * gw), yrow_b = raw + (uint32_t)((yt + 1 - ya) * gw);
    const uint32_t out_t = ring + (uint32_t)st * rowbytes, out_b = ring + (uint32_t)sb * rowbytes;
    const uint32_t uvrow = rawUV + (uint32_t)(u * gw);
    for (int q = lane; q < q4; q += 32) {
      const uint32_t uv = lds32(uvrow + 4 * q);
      const Chroma3 c0 = chroma_at<0>(uv, cm), c1 = chroma_at<16>(uv, cm);
      if (top) {
        const uint32_t yw = lds32(yrow_t + 4 * q);
        sts128(out_t + 16 * q, make_uint4(rgbx_dpx(byte_of<0>(yw), c0, cm), rgbx_dpx(byte_of<1>(yw), c0, cm),
                                          rgbx_dpx(byte_of<2>(yw), c1, cm), rgbx_dpx(byte_of<3>(yw), c1, cm)));
      }
      if (bot) {
        const uint32_t yw = lds32(yrow_b + 4 * q);
        sts128(out_b + 16 * q, make_uint4(rgbx_dpx(byte_of<0>(yw), c0, cm), rgbx_dpx(byte_of<1>(yw), c0, cm),
                                          rgbx_dpx(byte_of<2>(yw), c1, cm), rgbx_dpx(byte_of<3>(yw), c1, cm)));
      }
    }
  }
}

// convert_rows with the (UV row, 4-pixel group) units flattened over all threads of the CTA,
// so a row width that is not a multiple of 32 groups leaves no lane idle
__device__ __forceinline__ void convert_rows_flat(uint32_t ring, uint32_t raw, int gw, int ya, int yb, int y_first,
                                                  int ring_rows, uint32_t ring_magic, int tid, int nthr, const ColorM& cm) {
  const int ny = yb - ya + 1;
  if (ny <= 0) return;
  const int u0 = ya >> 1, nuv = (yb >> 1) - u0 + 1;
  const int q4 = gw >> 2;                      // 4-pixel groups per row
  const int total = nuv * q4;
  if (tid >= total) return;
  const uint32_t rawUV = raw + (uint32_t)(ny * gw);
  const uint32_t rowbytes = (uint32_t)gw * 4u;
  int u = tid / q4, q = tid - u * q4;          // unit -> (u, q), advanced incrementally
  const int du = nthr / q4, dq = nthr - du * q4;
  for (int i = tid; i < total; i += nthr) {
    const int yt = 2 * (u0 + u);
    const int st = (int)ring_mod((uint32_t)(yt - y_first + ring_rows), (uint32_t)ring_rows, ring_magic);
    const int sb = st + 1 == ring_rows ? 0 : st + 1;
    const uint32_t yrow_t = raw + (uint32_t)((yt - ya) * gw + 4 * q);
    const uint32_t uv = lds32(rawUV + (uint32_t)(u * gw + 4 * q));
    const Chroma3 c0 = chroma_at<0>(uv, cm), c1 = chroma_at<16>(uv, cm);
    if (yt >= ya) {
      const uint32_t yw = lds32(yrow_t);
      sts128(ring + (uint32_t)st * rowbytes + 16u * q,
             make_uint4(rgbx_dpx(byte_of<0>(yw), c0, cm), rgbx_dpx(byte_of<1>(yw), c0, cm), rgbx_dpx(byte_of<2>(yw), c1, cm),
                        rgbx_dpx(byte_of<3>(yw), c1, cm)));
    }
    if (yt + 1 <= yb) {
      const uint32_t yw = lds32(yrow_t + (uint32_t)gw);
      sts128(ring + (uint32_t)sb * rowbytes + 16u * q,
             make_uint4(rgbx_dpx(byte_of<0>(yw), c0, cm), rgbx_dpx(byte_of<1>(yw), c0, cm), rgbx_dpx(byte_of<2>(yw), c1, cm),
                        rgbx_dpx(byte_of<3>(yw), c1, cm)));
    }
    q += dq;
    u += du;
    if (q >= q4) {
      q -= q4;
      ++u;
    }
  }
}

// horizontal lerps of one ring row for the thread's column pair (R#12); col*: byte offsets
__device__ __forceinline__ void hrow_s(rs::Row3& r, uint32_t rowaddr, uint32_t ca0, uint32_t ca1, uint32_t cb0,
                                       uint32_t cb1, uint64_t lx) {
  const uint32_t a0 = lds32(rowaddr + ca0), a1 = lds32(rowaddr + ca1);
  const uint32_t b0 = lds32(rowaddr + cb0), b1 = lds32(rowaddr + cb1);
  r.h[0] = rs::hlerp<0>(a0, a1, b0, b1, lx);
  r.h[1] = rs::hlerp<1>(a0, a1, b0, b1, lx);
  r.h[2] = rs::hlerp<2>(a0, a1, b0, b1, lx);
}

// row actions of the walker (computed once per row by the table builder). Register sets hold
// the horizontal lerps of the output row's top (y0) and bottom (y1) source rows.
constexpr uint32_t kActTop = 1;    // (re)compute the top set from ring row y0
constexpr uint32_t kActBot = 2;    // (re)compute the bottom set from ring row y1
constexpr uint32_t kActFlip = 4;   // y0 = previous y0 + 1: the old bottom set becomes the top
// At the bottom edge (y1 == y0) the bottom set is not computed and lambda_y is stored as 0:
// fmaf(0, b - h0, h0) == h0 == fmaf(lambda, h0 - h0, h0) for any finite b (R#12 unchanged).

// Vertical lerp + rint + stores of one output row for NP (1 or 2) column pairs (R#12, R#17):
// 2 NP adjacent columns, one 4 NP-byte (bf16) / 8 NP-byte (f32) / 2 NP-byte (u8) store per
// channel and destination. Requires out_w % (2 NP) == 0 for every view (host-checked), so the
// stores are aligned.
// FOLD: the destinations' b fields hold b' = b - 2^23 a (ViewConst::fold) and the rint bias is
// 2^23: y = fmaf(2^23 + q, a, b') == fmaf(q, a, b) exactly, one packed add fewer per pair.
template <int DT, int ND, int NP, bool FOLD = false>
__device__ __forceinline__ void emit_np(const rs::Row3 (&top)[NP], const rs::Row3 (&bot)[NP], float l,
                                        rs::Dest (&dl)[ND], const LaunchParams& p, const uint32_t* __restrict__ dests,
                                        int nd, int oy, int ox) {
  static_assert(NP == 1 || NP == 2, "one or two column pairs");
  using namespace rs;
  const uint64_t ly = f2::splat(l);
  uint64_t q[NP][3], tq[NP][3];
#pragma unroll
  for (int j = 0; j < NP; ++j)
#pragma unroll
    for (int c = 0; c < 3; ++c) {
      const uint64_t dv = f2::fma(top[j].h[c], f2::splat(-1.f), bot[j].h[c]);   // h1 - h0
      const uint64_t v = f2::fma(ly, dv, top[j].h[c]);                          // fmaf(ly, h1-h0, h0)
      if constexpr (FOLD) {
        tq[j][c] = f2::add(v, f2::splat(kBias));                               // 2^23 + rint(v)
        q[j][c] = tq[j][c];
      } else {
        tq[j][c] = rint_biased(v);                                              // 1.5 * 2^23 + rint(v)
        q[j][c] = DT == SAND_U8 ? tq[j][c] : f2::add(tq[j][c], f2::splat(-kRound));
      }
    }
  auto store = [&](const Dest& d) {
#pragma unroll
    for (int c = 0; c < 3; ++c) {
      uint8_t* o = d.row + (size_t)c * d.cstride;
      if (DT == SAND_U8) {
        const uint32_t p0 = __byte_perm(f2::lo(tq[0][c]), f2::hi(tq[0][c]), 0x0040);
        if constexpr (NP == 2) {
          const uint32_t p1 = __byte_perm(f2::lo(tq[1][c]), f2::hi(tq[1][c]), 0x0040);
          *reinterpret_cast<uint32_t*>(o) = __byte_perm(p0, p1, 0x5410);
        } else {
          *reinterpret_cast<uint16_t*>(o) = (uint16_t)p0;
        }
      } else {
        const uint64_t a = f2::splat(d.a[c]), b = f2::splat(d.b[c]);
        const uint64_t y0 = f2::fma(q[0][c], a, b);                               // fmaf(q, a_c, b_c)
        if constexpr (NP == 2) {
          const uint64_t y1 = f2::fma(q[1][c], a, b);
          if (DT == SAND_BF16) {
            const __nv_bfloat162 v0 = __floats2bfloat162_rn(f2::lof(y0), f2::hif(y0));
            const __nv_bfloat162 v1 = __floats2bfloat162_rn(f2::lof(y1), f2::hif(y1));
            *reinterpret_cast<uint2*>(o) =
                make_uint2(*reinterpret_cast<const uint32_t*>(&v0), *reinterpret_cast<const uint32_t*>(&v1));
          } else {
            *reinterpret_cast<uint4*>(o) = make_uint4(f2::lo(y0), f2::hi(y0), f2::lo(y1), f2::hi(y1));
          }
        } else {
          if (DT == SAND_BF16) *reinterpret_cast<__nv_bfloat162*>(o) = __floats2bfloat162_rn(f2::lof(y0), f2::hif(y0));
          else *reinterpret_cast<uint64_t*>(o) = y0;
        }
      }
    }
  };
#pragma unroll
  for (int d = 0; d < ND; ++d) {
    if (d == 0 || d < nd) {
      store(dl[d]);
      dl[d].row += dl[d].rstride;
    }
  }
  for (int d = ND; d < nd; ++d) store(make_dest(p, dests[d], oy, ox, FOLD));   // rare: more destinations
}

}  // namespace st

// NP column pairs per thread: NP = 1 (any width, any dtype) or NP = 2 (out_w % 4 == 0 and a
// single specialised dtype; halves the per-row walker overhead per column)
#ifndef SAND_NP2_MINB
#define SAND_NP2_MINB 4   // resident 128-thread CTAs per SM the NP = 2 walker is compiled for
#endif
template <int DT, bool VEC, int NP>
__global__ void __launch_bounds__(NP == 1 ? 256 : 128, NP == 1 ? 3 : SAND_NP2_MINB) k_stream(const LaunchParams p, st::Shape sh, int maxWo) {
  static_assert(NP == 1 || (NP == 2 && VEC && DT >= 0), "NP = 2 needs the specialised vector path");
  extern __shared__ __align__(16) uint8_t smem_raw[];
  using namespace rs;
  const int tid = threadIdx.x, nthr = blockDim.x;
  const int warp = tid >> 5, lane = tid & 31;

  uint2* ctab = reinterpret_cast<uint2*>(smem_raw);
  uint4* rtab = reinterpret_cast<uint4*>(smem_raw + a16((size_t)maxWo * 8));
  uint32_t s_base = (uint32_t)__cvta_generic_to_shared(smem_raw);
  asm volatile("" : "+r"(s_base));   // materialise once: keeps the hot loops free of S2UR/LEA rebuilds
  const uint32_t s_rtab = s_base + (uint32_t)a16((size_t)maxWo * 8);
  const uint32_t s_ring = s_rtab + (uint32_t)a16((size_t)sh.SB * 16);
  const uint32_t s_raw = s_ring + (uint32_t)(sh.ring * sh.gw * 4);
  const uint32_t s_bar = s_raw + (uint32_t)a16((size_t)sh.raw_rows * sh.gw);   // staging mbarrier
  // persistent CTAs: task (item, super-band) indices blockIdx.x + i * gridDim.x (uniform
  // across the CTA, so item/group fields stay in uniform registers)
  const uint32_t n_tasks = p.n_items * (uint32_t)sh.nsb;
  if (tid == 0) {
    st::mbar_init(s_bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  uint32_t phase = 0;          // parity of the staging barrier's next completion

  for (uint32_t task = blockIdx.x; task < n_tasks; task += gridDim.x) {
  [&]() {
  const int item_idx = (int)(task / (uint32_t)sh.nsb);
  const int sb = (int)task - item_idx * sh.nsb;
  const WorkItem w = p.items[item_idx];
  if (w.flags & 1u) return;
  const GroupParams& g = p.groups[w.gp];
  const int Wo = g.out_w, Ho = g.out_h;
  const int Y0 = sb * sh.SB;
  if (Y0 >= Ho) return;
  const int nr = min(sh.SB, Ho - Y0);

  // footprint of the super-band (monotone taps)
  const int x_lo = tap0(g.sc_x, g.off_x, 0, g.org_x);
  int x_hi, dmy;
  float fl;
  tap(g.sc_x, g.off_x, Wo - 1, g.lim_x, g.org_x, dmy, x_hi, fl);
  const int x16 = x_lo & ~15;
  const int gw = ((x_hi + 16) & ~15) - x16;
  const uint32_t rowbytes = (uint32_t)gw * 4u;
  const int y_first = tap0(g.sc_y, g.off_y, Y0, g.org_y);
  const uint8_t* Yx = p.slab + w.y_off + x16;                // column x16 of Y row 0
  const uint8_t* UVx = Yx + (size_t)w.pitch * w.src_h;       // column x16 of UV row 0
  const uint32_t pitch = w.pitch;

  // sub-band k covers output rows [k*S, min((k+1)*S, nr)); it adds source rows
  // (y1(last row of k-1), y1(last row of k)]
  auto last_src = [&](int k) {
    int a, b;
    float l;
    tap(g.sc_y, g.off_y, Y0 + min((k + 1) * sh.S, nr) - 1, g.lim_y, g.org_y, a, b, l);
    return b;
  };
  const int nsub = (nr + sh.S - 1) / sh.S;
  int ya = y_first, yb = last_src(0);
  if (warp == 0) {
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // the previous task's generic reads of raw
    st::stage_rows(s_raw, s_bar, Yx, UVx, pitch, gw, ya, yb, lane, 32);
  }
  bool staged = true;          // sub-band k's rows were staged (k = 0 always adds rows)

  // tap tables (overlap the first copy): columns (x0, x1, lambda); rows (byte offsets of
  // the two ring rows, y0, lambda)
  for (int j = tid; j < Wo; j += nthr) {
    int x0, x1;
    float lx;
    tap(g.sc_x, g.off_x, j, g.lim_x, g.org_x, x0, x1, lx);
    ctab[j] = make_uint2((uint32_t)(x0 - x16) | ((uint32_t)(x1 - x16) << 16), __float_as_uint(lx));
  }
  for (int r = tid; r < nr; r += nthr) {
    int y0, y1;
    float ly;
    tap(g.sc_y, g.off_y, Y0 + r, g.lim_y, g.org_y, y0, y1, ly);
    const uint32_t s0 = st::ring_mod((uint32_t)(y0 - y_first), sh), s1 = st::ring_mod((uint32_t)(y1 - y_first), sh);
    // action relative to the previous output row of the super-band
    uint32_t act = st::kActTop | st::kActBot;      // first row or a step > 1
    if (r > 0) {
      const int yp = tap0(g.sc_y, g.off_y, Y0 + r - 1, g.org_y);
      act = y0 == yp ? 0u : (y0 == yp + 1 ? st::kActFlip | st::kActBot : act);
    }
    if (y1 == y0) {
      act &= ~st::kActBot;
      ly = 0.f;
    }
    rtab[r] = make_uint4(s0 * rowbytes, s1 * rowbytes, act, __float_as_uint(ly));
  }

  // per-thread walker state: output columns [ox, ox + 2 NP) for the whole super-band. Every
  // lane walks (lanes past the last column group repeat it without storing), so warps stay
  // converged.
  const int pairs = (Wo + 1) >> 1;
  const int ngrp = (pairs + NP - 1) / NP;
  int valid = tid < ngrp ? 1 : 0;
  asm volatile("" : "+r"(valid));   // keep it in a register: no TID re-read per row
  const int ox = 2 * NP * min(tid, ngrp - 1);
  const bool has_b = ox + 1 < Wo;
  const bool vec = has_b && !(Wo & 1);
  uint32_t ca0[NP], ca1[NP], cb0[NP], cb1[NP];
  uint64_t lx[NP];
  const int nd = (int)w.n_dest;
  const uint32_t* dests = p.dests + w.dest_begin;
  Dest dl[kInlineDests];
  int dt[kInlineDests];
  // Two register sets X, Y hold the horizontal lerps of source rows y0 and y0 + 1; `top`
  // says which one is y0. A shift by one source row flips `top` and recomputes only the other
  // set, so no register copies are needed between rows.
  Row3 X[NP], Y[NP];
#pragma unroll
  for (int j = 0; j < NP; ++j) {
    ca0[j] = ca1[j] = cb0[j] = cb1[j] = 0;
    lx[j] = 0ull;
#pragma unroll
    for (int c = 0; c < 3; ++c) X[j].h[c] = Y[j].h[c] = 0ull;   // finite (+0) before first use
  }
  int top = 0;
  auto hrows = [&](Row3 (&R)[NP], uint32_t rowaddr) {
#pragma unroll
    for (int j = 0; j < NP; ++j) st::hrow_s(R[j], rowaddr, ca0[j], ca1[j], cb0[j], cb1[j], lx[j]);
  };

  // One staging buffer: sub-band k+1's rows are copied while sub-band k is walked (the
  // copy is issued once the conversion of k has drained the buffer).
  for (int k = 0; k < nsub; ++k) {
    if (staged) {                                    // raw landed
      st::mbar_wait(s_bar, phase);
      phase ^= 1u;
    }
    __syncthreads();                                 // walk(k-1) finished: its ring rows are free
    if (staged) {
      if (sh.opts & 1) st::convert_rows(s_ring, s_raw, gw, ya, yb, y_first, sh.ring, sh.ring_magic, warp, nthr >> 5, lane, p.cm);
      else st::convert_rows_flat(s_ring, s_raw, gw, ya, yb, y_first, sh.ring, sh.ring_magic, tid, nthr, p.cm);
    }
    staged = false;
    __syncthreads();                                 // ring holds every row of sub-band k; raw drained
    if (k + 1 < nsub) {                              // stage the next sub-band's new rows
      const int na = yb + 1, nb = last_src(k + 1);
      if (nb >= na) {
        if (warp == 0) {
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");   // generic reads of raw before async writes
          st::stage_rows(s_raw, s_bar, Yx, UVx, pitch, gw, na, nb, lane, 32);
        }
        staged = true;
      }
      ya = na;
      yb = max(nb, yb);
    }
    if (k == 0) {                                    // tables are visible now
#pragma unroll
      for (int j = 0; j < NP; ++j) {
        const int oj = ox + 2 * j;                     // NP = 2: every pair is inside the row
        const bool hb = NP == 1 ? has_b : true;
        const int ja = g.flip ? Wo - 1 - oj : oj;
        const int jb = hb ? (g.flip ? Wo - 2 - oj : oj + 1) : ja;
        const uint2 ta = ctab[ja], tb = ctab[jb];
        ca0[j] = 4u * (ta.x & 0xffffu);
        ca1[j] = 4u * (ta.x >> 16);
        cb0[j] = 4u * (tb.x & 0xffffu);
        cb1[j] = 4u * (tb.x >> 16);
        lx[j] = f2::pack(ta.y, tb.y);
      }
#pragma unroll
      for (int d = 0; d < kInlineDests; ++d)
        if (d < nd) {
          dl[d] = make_dest(p, dests[d], Y0, ox);
          dt[d] = DT >= 0 ? DT : p.views[dests[d] >> 24].dtype;
        }
    }
    const int r_lo = k * sh.S, r_hi = min(r_lo + sh.S, nr);
    for (int rr = r_lo; rr < r_hi; ++rr) {
      const uint4 rt = st::lds128(s_rtab + 16u * rr);
      const uint32_t act = rt.z;
      const float l = __uint_as_float(rt.w);
      top ^= (act & st::kActFlip) ? 1 : 0;
      if (top == 0) {
        if (act & st::kActTop) hrows(X, s_ring + rt.x);
        if (act & st::kActBot) hrows(Y, s_ring + rt.y);
      } else {
        if (act & st::kActTop) hrows(Y, s_ring + rt.x);
        if (act & st::kActBot) hrows(X, s_ring + rt.y);
      }
      if (valid) {
        if constexpr (NP == 1) {
          if (top == 0) emit<DT, kInlineDests, VEC>(X[0], Y[0], l, dl, dt, p, dests, nd, Y0 + rr, ox, vec, has_b);
          else emit<DT, kInlineDests, VEC>(Y[0], X[0], l, dl, dt, p, dests, nd, Y0 + rr, ox, vec, has_b);
        } else {
          if (top == 0) st::emit_np<DT, kInlineDests, NP>(X, Y, l, dl, p, dests, nd, Y0 + rr, ox);
          else st::emit_np<DT, kInlineDests, NP>(Y, X, l, dl, p, dests, nd, Y0 + rr, ox);
        }
      }
    }
  }
  }();
  __syncthreads();             // task done: shared memory free for the next one
  }
}

}  // namespace sand
