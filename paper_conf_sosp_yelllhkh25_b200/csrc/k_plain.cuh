// k_plain.cuh — multi-frame streaming resample kernel for plain items (no rotation / blur)
// with mild scaling (source step <= 2 rows and columns per output row / column): Kinetics RRC,
// SlowFast short-side crops with real scaling, two-view plain groups, tiny (SURVEY §8(a)
// a4-a7, a10, a11).
//
// A TASK is (run of up to FPC items of ONE (clip slot, spatial group), band of output rows).
// Spatial parameters are per clip and group (R#7), so the FPC frames of a task share every tap,
// table and branch: the CTA holds FPC x NQ threads (NQ = output columns per row / (2 NP), NP
// column pairs per thread; 4 x 112 = 448 for 224-wide outputs at NP = 1, no idle lanes) whose
// control flow is identical, each frame with its
// own source rows in shared memory. The band's source rows [y_first, y_last] are walked in
// CHUNKS of CR rows (chunk boundaries at even rows, so a UV row never straddles two chunks):
//   * the NV12 rows of chunks j + 1 and j + 2 are copied HBM -> shared memory by the TMA engine
//     (cp.async.bulk, one copy per row per frame, completion counted on the staging buffer's
//     mbarrier; two staging buffers) while chunk j is converted and walked (a4);
//   * chunk j is converted once into RGBx rows (R#11, the DPX formulation of k_stream.cuh; a5):
//     each thread owns fixed (frame, 4-pixel group) slots and converts their UV rows;
//   * the walk is SOURCE-ROW major: each thread owns 2 NP adjacent output columns of its frame,
//     computes the horizontal lerps of each source row once (R#12, a6; flip mirrors the column
//     taps, a7) into one of two register sets whose roles alternate with the row's parity
//     (static in the unrolled code: no register copies), and emits every output row whose top
//     tap is the previous source row: vertical lerp, rint, normalise and 4 NP-byte (bf16)
//     stores per channel to every destination view of the item (a10, a11).
// Every fp32 operation is the R#12/R#17 op sequence with IEEE rounding: bit-identical to the
// oracle. Tasks and the exact staged span are computed on the host from the same fp32 tap rule
// (view.cpp).
#pragma once

namespace sand {
namespace pl {

#ifndef SAND_PL_CR
#define SAND_PL_CR 8
#endif
#ifndef SAND_PL_MINB
#define SAND_PL_MINB 2
#endif
constexpr int kCR = SAND_PL_CR;       // source rows per chunk (even)
constexpr int kRawRows = kCR + kCR / 2 + 1;   // staging rows per chunk: Y rows + their UV rows

struct Shape {        // host-chosen launch shape of one batch's plain items
  int fpc;            // frames (items of one run) per CTA
  int nq;             // threads per frame = output columns of the widest view / (2 NP)
  int rb;             // largest band (rows of the row table)
  int gw;             // row capacity in pixels (multiple of 16, >= every item's staged span)
};

// per frame: the converted rows of one chunk, then two staging buffers
__host__ __device__ inline size_t conv_bytes(const Shape& s) { return (size_t)kCR * s.gw * 4; }
__host__ __device__ inline size_t raw_bytes(const Shape& s) { return rs::a16((size_t)kRawRows * s.gw); }
__host__ __device__ inline size_t frame_bytes(const Shape& s) { return conv_bytes(s) + 2 * raw_bytes(s); }
__host__ __device__ inline size_t smem_bytes(const Shape& s) {
  return rs::a16((size_t)s.rb * 8) + 16 + (size_t)s.fpc * frame_bytes(s);
}

// task encoding (uint2, built by view.cpp): x = first item (index into the launch's items),
// y = pl_task_y(frames, band rows, first output row) (plan_types.h)

// exact quotient of small non-negative integers r / n via a float reciprocal (r < 2^16, n < 2^12)
__device__ __forceinline__ int small_div(int r, float inv_n) { return (int)(((float)r + 0.5f) * inv_n); }

}  // namespace pl

// NP column pairs per thread (1: 2 columns, 448-thread CTAs of 14 warps; 2: 4 columns)
template <int NP>
struct PlainBounds {
  static constexpr int kThreads = NP == 1 ? 448 : 224;
  static constexpr int kMinBlocks = SAND_PL_MINB;
};

template <int DT, int ND, int NP, bool FOLD>
__global__ void __launch_bounds__(PlainBounds<NP>::kThreads, PlainBounds<NP>::kMinBlocks) k_plain(const LaunchParams p, const uint2* __restrict__ tasks, pl::Shape sh) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  using namespace rs;
  using pl::kCR;
  const int tid = threadIdx.x, nthr = blockDim.x;
  const int warp = tid >> 5, lane = tid & 31;
  const uint2 tk = tasks[blockIdx.x];
  const int item0 = (int)tk.x;
  const int nfr = (int)(tk.y & 0xffu), nr = (int)((tk.y >> 8) & 0xfffu), Y0 = (int)(tk.y >> 20);
  const WorkItem w0 = p.items[item0];
  const GroupParams& g = p.groups[w0.gp];
  const int Wo = g.out_w;
  const float sc_x = g.sc_x, sc_y = g.sc_y;
  const int off_x = g.off_x, off_y = g.off_y, org_x = g.org_x, org_y = g.org_y;
  const int lim_x = g.lim_x, lim_y = g.lim_y, flip = g.flip;
  const ColorM cm = p.cm;                                          // YUV -> RGB matrix (R#11 / R#29)

  uint32_t s_base = (uint32_t)__cvta_generic_to_shared(smem_raw);
  asm volatile("" : "+r"(s_base));
  const uint32_t s_tab = s_base;                                   // rb x 8 B row table
  const uint32_t s_bar = s_tab + (uint32_t)a16((size_t)sh.rb * 8);  // two mbarriers (staging buffers)
  const uint32_t s_fr = s_bar + 16;                                // frame f at s_fr + f * fbytes
  const uint32_t fbytes = (uint32_t)pl::frame_bytes(sh);
  const uint32_t rowbytes = (uint32_t)sh.gw * 4u;                  // converted row stride
  const uint32_t raw_off = (uint32_t)pl::conv_bytes(sh);           // staging buffer b at raw_off + b * rawb
  const uint32_t rawb = (uint32_t)pl::raw_bytes(sh);
  const uint32_t rawpitch = (uint32_t)sh.gw;                       // staging row stride

  // staged column span (monotone taps): [x16, x16 + gwi)
  const int x_lo = tap0(sc_x, off_x, 0, org_x);
  int x_hi, dmy;
  float fl;
  tap(sc_x, off_x, Wo - 1, lim_x, org_x, dmy, x_hi, fl);
  const int x16 = x_lo & ~15;
  const int gwi = ((x_hi + 16) & ~15) - x16;
  if (gwi > sh.gw) __trap();                                       // host bound violated (never)
  // source rows of the band: y0 of its first row .. y1 of its last row (monotone taps)
  const int y_first = tap0(sc_y, off_y, Y0, org_y);
  int y_last;
  tap(sc_y, off_y, Y0 + nr - 1, lim_y, org_y, dmy, y_last, fl);
  const int ybase = y_first & ~1;                                  // chunk j: [ybase + j CR, + CR)
  const int nchunks = (y_last - ybase) / kCR + 1;

  if (tid == 0) {
    st::mbar_init(s_bar, 1);
    st::mbar_init(s_bar + 8, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  auto chunk_lo = [&](int j) { return max(y_first, ybase + j * kCR); };
  auto chunk_hi = [&](int j) { return min(y_last, ybase + j * kCR + kCR - 1); };
  // chunk j's NV12 rows (Y rows, then their UV rows) of every frame -> staging buffer j & 1, one
  // bulk copy per row, completion counted on that buffer's mbarrier (warp 0)
  auto stage = [&](int j) {
    const int ya = chunk_lo(j), yb = chunk_hi(j);
    const int ny = yb - ya + 1, u0 = ya >> 1, nuv = (yb >> 1) - u0 + 1, per = ny + nuv;
    const uint32_t bar = s_bar + 8u * (uint32_t)(j & 1);
    const uint32_t dst0 = s_fr + raw_off + (uint32_t)(j & 1) * rawb;
    if (lane == 0) st::mbar_arrive_expect_tx(bar, (uint32_t)(nfr * per * gwi));
    const float inv = 1.0f / (float)per;
    for (int c = lane; c < nfr * per; c += 32) {
      const int f = pl::small_div(c, inv), r = c - f * per;
      const WorkItem& w = p.items[item0 + f];
      const uint8_t* src = p.slab + w.y_off + x16 +
                           (r < ny ? (size_t)(ya + r) * w.pitch : (size_t)w.pitch * (w.src_h + u0 + r - ny));
      st::bulk_g2s(dst0 + (uint32_t)f * fbytes + (uint32_t)r * rawpitch, src, (uint32_t)gwi, bar);
    }
  };
  if (warp == 0) {
    stage(0);
    if (nchunks > 1) stage(1);
  }

  // row table: (y0 of the output row, lambda_y); lambda 0 at the bottom clamp (y1 == y0), where
  // the row is emitted from (H(y0), H(y0)): fmaf(0, h - h, h) == h (R#12 unchanged)
  for (int r = tid; r < nr; r += nthr) {
    int y0, y1;
    float ly;
    tap(sc_y, off_y, Y0 + r, lim_y, org_y, y0, y1, ly);
    if (y1 == y0) ly = 0.f;
    asm volatile("st.shared.v2.u32 [%0], {%1, %2};" ::"r"(s_tab + 8u * (uint32_t)r), "r"((uint32_t)y0),
                 "r"(__float_as_uint(ly))
                 : "memory");
  }

  // walker: frame f, output columns [ox, ox + 2 NP)
  const int f = tid / sh.nq;
  const int qd = tid - f * sh.nq;
  const int ox = 2 * NP * qd;
  int active = (f < nfr && ox < Wo) ? 1 : 0;
  asm volatile("" : "+r"(active));
  const int fa = min(f, nfr - 1);
  const uint32_t rowsf = s_fr + (uint32_t)fa * fbytes;             // this frame's conversion buffers
  uint32_t ca0[NP], ca1[NP], cb0[NP], cb1[NP];
  uint64_t lx[NP];
#pragma unroll
  for (int j = 0; j < NP; ++j) {
    const int oj = min(ox + 2 * j, Wo - 2);
    const int ja = flip ? Wo - 1 - oj : oj;
    const int jb = flip ? Wo - 2 - oj : oj + 1;
    int a0, a1, b0, b1;
    float la, lb;
    tap(sc_x, off_x, ja, lim_x, org_x, a0, a1, la);
    tap(sc_x, off_x, jb, lim_x, org_x, b0, b1, lb);
    // shared addresses of the four taps in this frame's conversion buffer 0, row slot 0; a row
    // is then one offset common to the whole CTA (uniform)
    ca0[j] = rowsf + 4u * (uint32_t)(a0 - x16);
    ca1[j] = rowsf + 4u * (uint32_t)(a1 - x16);
    cb0[j] = rowsf + 4u * (uint32_t)(b0 - x16);
    cb1[j] = rowsf + 4u * (uint32_t)(b1 - x16);
    lx[j] = f2::pack(__float_as_uint(la), __float_as_uint(lb));
  }
  const WorkItem wf = p.items[item0 + fa];
  const int nd = (int)wf.n_dest;
  const uint32_t* dests = p.dests + wf.dest_begin;
  Dest dl[ND];
#pragma unroll
  for (int d = 0; d < ND; ++d) dl[d] = make_dest(p, dests[d < nd ? d : 0], Y0, ox, FOLD);
  Row3 X[NP], Y[NP];
#pragma unroll
  for (int j = 0; j < NP; ++j)
#pragma unroll
    for (int c = 0; c < 3; ++c) X[j].h[c] = Y[j].h[c] = 0ull;
  auto hrows = [&](Row3 (&R)[NP], uint32_t rowoff) {
#pragma unroll
    for (int j = 0; j < NP; ++j) st::hrow_s(R[j], rowoff, ca0[j], ca1[j], cb0[j], cb1[j], lx[j]);
  };
  int r = 0;                               // next output row to emit
  uint2 rt = make_uint2(0xffffffffu, 0u);  // its table entry (y0, lambda)
  // emit every output row whose y0 is `y` from the lerps of rows y (T) and y + 1 (B)
  auto emit_rows = [&](const Row3 (&T)[NP], const Row3 (&B)[NP], int y) {
    while ((int)rt.x == y) {
      if (active) st::emit_np<DT, ND, NP, FOLD>(T, B, __uint_as_float(rt.y), dl, p, dests, nd, Y0 + r, ox);
      ++r;
      rt.x = 0xffffffffu;
      if (r < nr) asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(rt.x), "=r"(rt.y) : "r"(s_tab + 8u * (uint32_t)r));
    }
  };

  // conversion slots: (frame, 4-pixel group) pairs, fixed per thread for the whole task (thread t
  // owns slots t, t + nthr, ...); a chunk converts every UV row of every slot
  const int q4 = gwi >> 2;
  const int n_slots = nfr * q4;
  // chunk j: staged rows -> RGBx rows of the conversion buffer, after waiting for its staging buffer
  auto convert = [&](int j) {
    const int ya = chunk_lo(j), yb = chunk_hi(j);
    st::mbar_wait(s_bar + 8u * (uint32_t)(j & 1), (uint32_t)(j >> 1) & 1u);
    const int ny = yb - ya + 1, u0 = ya >> 1, nuv = (yb >> 1) - u0 + 1;
    const uint32_t slot0 = (uint32_t)(ybase + j * kCR);            // absolute row of slot 0
    const uint8_t* rawb0 = smem_raw + (s_fr - s_base) + raw_off + (uint32_t)(j & 1) * rawb;
    uint8_t* convb0 = smem_raw + (s_fr - s_base);
#if SAND_PL_FLAT
    // units = (frame, UV row, 4-pixel group), flattened over the CTA (balanced)
    const int upf = nuv * q4;
    const float inv_upf = 1.0f / (float)upf, inv_q4 = 1.0f / (float)q4;
    for (int i = tid; i < nfr * upf; i += nthr) {
      const int fr = pl::small_div(i, inv_upf), rem = i - fr * upf;
      const int u = pl::small_div(rem, inv_q4), q = rem - u * q4;
      const uint8_t* raw = rawb0 + (uint32_t)fr * fbytes + 4u * q;
      uint8_t* conv = convb0 + (uint32_t)fr * fbytes + 16u * q;
      const int yt = 2 * (u0 + u);
      const uint32_t uv = *reinterpret_cast<const uint32_t*>(raw + (uint32_t)(ny + u) * rawpitch);
      const st::Chroma3 c0 = st::chroma_at<0>(uv, cm), c1 = st::chroma_at<16>(uv, cm);
      uint8_t* out = conv + ((uint32_t)yt - slot0) * rowbytes;
      if (yt >= ya) {
        const uint32_t yw = *reinterpret_cast<const uint32_t*>(raw + (uint32_t)(yt - ya) * rawpitch);
        *reinterpret_cast<uint4*>(out) = make_uint4(st::rgbx_dpx(st::byte_of<0>(yw), c0, cm), st::rgbx_dpx(st::byte_of<1>(yw), c0, cm),
                                                    st::rgbx_dpx(st::byte_of<2>(yw), c1, cm), st::rgbx_dpx(st::byte_of<3>(yw), c1, cm));
      }
      if (yt + 1 <= yb) {
        const uint32_t yw = *reinterpret_cast<const uint32_t*>(raw + (uint32_t)(yt + 1 - ya) * rawpitch);
        *reinterpret_cast<uint4*>(out + rowbytes) =
            make_uint4(st::rgbx_dpx(st::byte_of<0>(yw), c0, cm), st::rgbx_dpx(st::byte_of<1>(yw), c0, cm),
                       st::rgbx_dpx(st::byte_of<2>(yw), c1, cm), st::rgbx_dpx(st::byte_of<3>(yw), c1, cm));
      }
    }
#else
    for (int sl = tid; sl < n_slots; sl += nthr) {
      const int fr = sl / q4, q = sl - fr * q4;
      const uint8_t* raw = rawb0 + (uint32_t)fr * fbytes + 4u * q;
      uint8_t* conv = convb0 + (uint32_t)fr * fbytes + 16u * q;
      for (int u = 0; u < nuv; ++u) {
        const int yt = 2 * (u0 + u);                       // top Y row of this UV row
        const uint32_t uv = *reinterpret_cast<const uint32_t*>(raw + (uint32_t)(ny + u) * rawpitch);
        const st::Chroma3 c0 = st::chroma_at<0>(uv, cm), c1 = st::chroma_at<16>(uv, cm);
        uint8_t* out = conv + ((uint32_t)yt - slot0) * rowbytes;   // row yt
        if (yt >= ya) {
          const uint32_t yw = *reinterpret_cast<const uint32_t*>(raw + (uint32_t)(yt - ya) * rawpitch);
          *reinterpret_cast<uint4*>(out) = make_uint4(st::rgbx_dpx(st::byte_of<0>(yw), c0, cm), st::rgbx_dpx(st::byte_of<1>(yw), c0, cm),
                                                      st::rgbx_dpx(st::byte_of<2>(yw), c1, cm), st::rgbx_dpx(st::byte_of<3>(yw), c1, cm));
        }
        if (yt + 1 <= yb) {
          const uint32_t yw = *reinterpret_cast<const uint32_t*>(raw + (uint32_t)(yt + 1 - ya) * rawpitch);
          *reinterpret_cast<uint4*>(out + rowbytes) =
              make_uint4(st::rgbx_dpx(st::byte_of<0>(yw), c0, cm), st::rgbx_dpx(st::byte_of<1>(yw), c0, cm),
                         st::rgbx_dpx(st::byte_of<2>(yw), c1, cm), st::rgbx_dpx(st::byte_of<3>(yw), c1, cm));
        }
      }
    }
#endif
  };
  // walk of chunk j: source row y's lerps go to X when (y - y_first) is even, else to Y; the
  // output rows whose top tap is y - 1 are emitted as soon as y's lerps exist
  auto walk = [&](int j) {
    const int ya = chunk_lo(j), yb = chunk_hi(j);
    uint32_t row = (uint32_t)(ya - ybase - j * kCR) * rowbytes;   // offset of row ya
    int y = ya;
    if ((y - y_first) & 1) {
      hrows(Y, row);
      emit_rows(X, Y, y - 1);
      ++y;
      row += rowbytes;
    }
    for (; y + 1 <= yb; y += 2) {
      hrows(X, row);
      emit_rows(Y, X, y - 1);
      hrows(Y, row + rowbytes);
      emit_rows(X, Y, y);
      row += 2 * rowbytes;
    }
    if (y <= yb) {
      hrows(X, row);
      emit_rows(Y, X, y - 1);
    }
  };

  // single-buffered chunks: convert chunk j, barrier, stage chunk j + 1, walk chunk j
  for (int j = 0; j < nchunks; ++j) {
    __syncthreads();                       // walk of chunk j - 1 done: conversion buffer free
    convert(j);
    __syncthreads();                       // chunk j converted, its staging buffer drained
    if (j == 0) asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(rt.x), "=r"(rt.y) : "r"(s_tab));
    if (j + 2 < nchunks && warp == 0) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      stage(j + 2);
    }
    walk(j);
  }
  // rows at the bottom clamp (y0 == y1 == y_last, lambda 0): emitted from H(y_last) twice
  if ((y_last - y_first) & 1) emit_rows(Y, Y, y_last);
  else emit_rows(X, X, y_last);
}

}  // namespace sand
