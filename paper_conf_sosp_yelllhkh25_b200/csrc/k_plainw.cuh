// k_plainw.cuh — frame-group resample kernel for plain items with mild scaling (source step <= 2:
// Kinetics RRC, two-view plain groups, short-side crops with real scaling; SURVEY §8(a) a4-a7,
// a10, a11).
//
// A task is (up to 8 frames of ONE (clip slot, group), band of <= kMaxRB output rows), as for k_plain;
// a CTA serves kFrames of its frames. Each frame is served by a FRAME GROUP of two warps that synchronise
// only with each other (named barrier 1 + frame, 64 threads), never with the rest of the CTA:
//   * the group stages its frame's source rows in QUADS (four Y rows from an even row and their
//     two UV rows), one TMA bulk copy (`cp.async.bulk`) per row into a ring of kStages quads,
//     completion counted on the stage's mbarrier (a4);
//   * both warps convert a staged quad into four RGBx rows (R#11 / R#29, the DPX form of
//     k_stream.cuh), 64 lanes over (UV row, 4-pixel group) units, into one of two RGBx buffers
//     (double-buffered: one group barrier per quad) (a5);
//   * each warp walks HALF of the output columns SOURCE-ROW major: the horizontal lerps of each
//     source row are computed once (R#12, a6; flip mirrors the column taps, a7) into the
//     register set of the row's parity, and every output row whose top tap is the previous
//     source row is emitted at once: vertical lerp, rint, normalise and stores to every
//     destination view (a10, a11).
// Lane L of half h owns the column pairs (h Wo/2 + 2L + 64j, + 1), j < NPJ: neighbouring lanes
// read neighbouring converted pixels and every store instruction of the warp writes one
// contiguous 128-byte (bf16) row segment. The output-row table (y0, lambda_y) of the band is in
// shared memory with a sentinel entry. Every fp32 operation is the R#12 / R#17 op sequence with
// IEEE rounding: bit-identical to the oracle.
#pragma once

#ifndef SAND_PW_MINB
#define SAND_PW_MINB 5
#endif

namespace sand {
namespace pw {

#ifndef SAND_PW_STAGES
#define SAND_PW_STAGES 3
#endif
constexpr int kStages = SAND_PW_STAGES;   // NV12 row quads in flight per frame
#ifndef SAND_PW_GWMAX
#define SAND_PW_GWMAX 384
#endif
constexpr int kGWMax = SAND_PW_GWMAX;     // widest staged span (pixels); wider tasks take k_plain
static_assert(kGWMax == kPlainwMaxSpan, "the host partitions tasks at kPlainwMaxSpan");
constexpr int kRow = 4 * kGWMax;          // byte stride of the converted RGBx rows
constexpr int kFrames = 2;                // frames per CTA (two warps each: 128 threads)
constexpr int kMaxRB = 64;                // output rows per band (task) at most
constexpr uint32_t kTabBytes = (8u * (kMaxRB + 1) + 15u) & ~15u;   // output-row table + sentinel
constexpr uint32_t kBarBytes = (8u * kStages + 15u) & ~15u;   // the stages' mbarriers

struct Shape {
  int nsub;  // CTAs per task: CTA s of a task serves its frames [kFrames s, kFrames (s + 1))
  int gw;    // staged row capacity in pixels (multiple of 16, >= every item's span, <= kGWMax)
};

// per frame: two RGBx buffers of four rows, kStages x (4 Y + 2 UV) staging rows, kStages
// mbarriers, the output-row table
__host__ __device__ inline uint32_t stage_bytes(int gw) { return 6u * (uint32_t)gw; }
__host__ __device__ inline uint32_t frame_bytes(int gw) {
  return 8u * kRow + kStages * stage_bytes(gw) + kBarBytes + kTabBytes;   // a multiple of 16
}
__host__ __device__ inline size_t smem_bytes(const Shape& s) { return (size_t)kFrames * frame_bytes(s.gw); }

// named barrier 1 + f of frame group f (immediate ids: a register id would reserve all 16)
__device__ __forceinline__ void group_sync(int f) {
  if (f == 0) asm volatile("bar.sync 1, 64;" ::: "memory");
  else asm volatile("bar.sync 2, 64;" ::: "memory");
}

}  // namespace pw

template <int DT, int ND, int NPJ, bool FOLD>
__global__ void __launch_bounds__(128, SAND_PW_MINB) k_plainw(const LaunchParams p, const uint2* __restrict__ tasks,
                                                               pw::Shape sh) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  using namespace rs;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int fr = warp >> 1, half = warp & 1, gt = threadIdx.x & 63;   // frame, half, thread in group
  // the next batch's kernel may launch once every CTA of this one is resident: its prologue then
  // overlaps this grid's tail (it waits for this grid before touching frames or outputs)
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  const int task = (int)blockIdx.x / sh.nsub, sub = (int)blockIdx.x - task * sh.nsub;
  const uint2 tk = tasks[task];
  const int nfr = (int)(tk.y & 0xffu), nr = (int)((tk.y >> 8) & 0xfffu), Y0 = (int)(tk.y >> 20);
  const int fi = pw::kFrames * sub + fr;                           // frame of the task
  if (fi >= nfr) return;                                           // only group barriers follow
  const WorkItem w = p.items[tk.x + fi];
  const GroupParams& g = p.groups[w.gp];
  const int Wo = g.out_w;
  const float sc_x = g.sc_x, sc_y = g.sc_y;
  const int off_x = g.off_x, off_y = g.off_y, org_x = g.org_x, org_y = g.org_y;
  const int lim_x = g.lim_x, lim_y = g.lim_y, flip = g.flip;
  const ColorM cm = p.cm;
  const int Wh = Wo >> 1, c0 = half * Wh;                          // this warp's columns [c0, c0 + Wh)

  uint32_t s_f = (uint32_t)__cvta_generic_to_shared(smem_raw) + (uint32_t)fr * pw::frame_bytes(sh.gw);
  asm volatile("" : "+r"(s_f));
  const uint32_t gw = (uint32_t)sh.gw;
  const uint32_t stb = pw::stage_bytes(sh.gw);
  const uint32_t s_rgb = s_f;                                      // buffer b, row i at + (4b + i) kRow
  const uint32_t s_stage = s_f + 8u * pw::kRow;                    // stage s at + s stb: Y0..Y3, UV0, UV1
  const uint32_t s_bar = s_stage + pw::kStages * stb;              // mbarrier of stage s at + 8 s
  const uint32_t s_tab = s_bar + pw::kBarBytes;                   // row table (nr + 1 entries of 8 B)

  // staged column span [x16, x16 + gwi) of the whole frame row (monotone taps)
  const int x_lo = tap0(sc_x, off_x, 0, org_x);
  int x_hi, dmy;
  float fl;
  tap(sc_x, off_x, Wo - 1, lim_x, org_x, dmy, x_hi, fl);
  const int x16 = x_lo & ~15;
  const int gwi = ((x_hi + 16) & ~15) - x16;
  if (gwi > sh.gw) __trap();                                       // host bound violated (never)

  // output-row table (warp 0 of the group): entry r = row Y0 + r's (y0, lambda); lambda 0 at the
  // bottom clamp (y1 == y0), where the row is emitted from (H(y0), H(y0)): fmaf(0, h - h, h) == h;
  // entry nr is a sentinel
  if (half == 0) {
    for (int r = lane; r <= nr; r += 32) {
      uint32_t e0 = 0x7fffffffu, e1 = 0u;
      if (r < nr) {
        int a, b;
        float l;
        tap(sc_y, off_y, Y0 + r, lim_y, org_y, a, b, l);
        e0 = (uint32_t)a;
        e1 = __float_as_uint(b == a ? 0.f : l);
      }
      asm volatile("st.shared.v2.u32 [%0], {%1, %2};" ::"r"(s_tab + 8u * r), "r"(e0), "r"(e1) : "memory");
    }
  }
  const int y_first = tap0(sc_y, off_y, Y0, org_y);
  int y_last;
  tap(sc_y, off_y, Y0 + nr - 1, lim_y, org_y, dmy, y_last, fl);
  const int ybase = y_first & ~1;
  const int nquads = ((y_last - ybase) >> 2) + 1;

  const uint8_t* ysrc = p.slab + w.y_off + x16;                    // column x16 of Y row 0
  const uint8_t* uvsrc = ysrc + (size_t)w.pitch * w.src_h;         // column x16 of UV row 0
  const uint32_t pitch = w.pitch;
  // quad k (Y rows ybase + 4k .. + 3 inside [y_first, y_last] and their UV rows) -> stage
  // k % kStages by one warp of the group (the first kStages quads: warp 0; then the warps take
  // turns), lanes 0..5 one row copy each (the mbarrier's tx-count may go transiently negative
  // before lane 0's expect)
  auto stage = [&](int k) {
    const int yq = ybase + 4 * k;
    const int ya = max(yq, y_first), yb = min(yq + 3, y_last);
    const int nuv = ((yb >> 1) - (ya >> 1)) + 1;
    const uint32_t si = (uint32_t)(k % pw::kStages);
    const uint32_t bar = s_bar + 8u * si;
    if (lane == 0) st::mbar_arrive_expect_tx(bar, (uint32_t)((yb - ya + 1 + nuv) * gwi));
    const int y = yq + lane, u = (yq >> 1) + lane - 4;
    const bool cp = lane < 4 ? (y >= ya && y <= yb) : (lane < 6 && u >= (ya >> 1) && u <= (yb >> 1));
    if (cp) {
      const uint8_t* src = lane < 4 ? ysrc + (size_t)y * pitch : uvsrc + (size_t)u * pitch;
      st::bulk_g2s(s_stage + si * stb + (uint32_t)lane * gw, src, (uint32_t)gwi, bar);
    }
  };
  if (half == 0) {
    if (lane == 0) {
#pragma unroll
      for (int s = 0; s < pw::kStages; ++s) st::mbar_init(s_bar + 8u * s, 1);
      asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
  }

  // column taps of the lane's pairs: shared addresses of tap i0 in RGBx row 0 of the current
  // quad's buffer (rebased per quad; tap i1 is the next word; at the right clamp i1 == i0 lambda
  // is 0 instead, fmaf(0, d, p0) == p0)
  uint32_t ca[NPJ], cb[NPJ];
  uint64_t lx[NPJ];
#pragma unroll
  for (int j = 0; j < NPJ; ++j) {
    const int oa = c0 + min(2 * lane + 64 * j, Wh - 2);
    const int ja = flip ? Wo - 1 - oa : oa;
    const int jb = flip ? Wo - 2 - oa : oa + 1;
    int a0, a1, b0, b1;
    float la, lb;
    tap(sc_x, off_x, ja, lim_x, org_x, a0, a1, la);
    tap(sc_x, off_x, jb, lim_x, org_x, b0, b1, lb);
    if (a1 == a0) la = 0.f;
    if (b1 == b0) lb = 0.f;
    ca[j] = s_rgb + 4u * (uint32_t)(a0 - x16);
    cb[j] = s_rgb + 4u * (uint32_t)(b0 - x16);
    lx[j] = f2::pack(__float_as_uint(la), __float_as_uint(lb));
  }
  // pair j of the lane is a real column pair (NPJ = 2 is used for Wh > 64: pair 0 always is)
  bool act[NPJ];
#pragma unroll
  for (int j = 0; j < NPJ; ++j) act[j] = (NPJ == 2 && j == 0) || 2 * lane + 64 * j < Wh;
  const int nd = (int)w.n_dest;                                   // <= ND (host-checked)
  const uint32_t* dests = p.dests + w.dest_begin;
  // destinations kept in registers: one row pointer per channel plane, advanced per row
  struct DestC {
    uint8_t* o[3];
    uint32_t rstride;
    float a[3], b[3];
  };
  DestC dl[ND];
#pragma unroll
  for (int d = 0; d < ND; ++d) {
    const Dest e = make_dest(p, dests[d < nd ? d : 0], Y0, c0 + 2 * lane, FOLD);
#pragma unroll
    for (int c = 0; c < 3; ++c) {
      dl[d].o[c] = e.row + (size_t)c * e.cstride;
      dl[d].a[c] = e.a[c];
      dl[d].b[c] = e.b[c];
    }
    dl[d].rstride = e.rstride;
  }

  // Programmatic dependent launch (mat_plain.cu): everything above reads only this batch's plan
  // (uploaded and ordered before the launch); frames and outputs are touched only after the
  // previous kernel on the stream has completed (a no-op when the launch is not programmatic)
  asm volatile("griddepcontrol.wait;" ::: "memory");
  if (half == 0) {
    __syncwarp();
    for (int k = 0; k < min(nquads, pw::kStages); ++k) stage(k);
  }

  Row3 X[NPJ], Yr[NPJ];                                            // lerps of even / odd source rows
#pragma unroll
  for (int j = 0; j < NPJ; ++j)
#pragma unroll
    for (int c = 0; c < 3; ++c) X[j].h[c] = Yr[j].h[c] = 0ull;
  auto hrows = [&](Row3 (&R)[NPJ], uint32_t rowoff) {
#pragma unroll
    for (int j = 0; j < NPJ; ++j) {
      const uint32_t a0 = st::lds32(ca[j] + rowoff), a1 = st::lds32(ca[j] + rowoff + 4u);
      const uint32_t b0 = st::lds32(cb[j] + rowoff), b1 = st::lds32(cb[j] + rowoff + 4u);
      R[j].h[0] = hlerp<0>(a0, a1, b0, b1, lx[j]);
      R[j].h[1] = hlerp<1>(a0, a1, b0, b1, lx[j]);
      R[j].h[2] = hlerp<2>(a0, a1, b0, b1, lx[j]);
    }
  };

  // one output row from the lerps of its top (T) and bottom (B) source rows
  auto emit = [&](const Row3 (&T)[NPJ], const Row3 (&B)[NPJ], float l) {
    const uint64_t ly = f2::splat(l);
    // channel c of pair j: quantised pair (2^23 or 1.5 * 2^23 + rint(v)), stored to plane o
    auto put = [&](uint8_t* o, float a_c, float b_c, int j, uint64_t q) {
      if (DT == SAND_U8) {
        const uint16_t v = (uint16_t)__byte_perm(f2::lo(q), f2::hi(q), 0x0040);
        if (act[j]) *reinterpret_cast<uint16_t*>(o + 64 * j) = v;
      } else {
        const uint64_t qq = FOLD ? q : f2::add(q, f2::splat(-kRound));
        const uint64_t y = f2::fma(qq, f2::splat(a_c), f2::splat(b_c));   // fmaf(q, a_c, b_c)
        if (DT == SAND_BF16) {
          const __nv_bfloat162 v = __floats2bfloat162_rn(f2::lof(y), f2::hif(y));
          if (act[j]) *reinterpret_cast<__nv_bfloat162*>(o + 128 * j) = v;
        } else {
          if (act[j]) *reinterpret_cast<uint64_t*>(o + 256 * j) = y;
        }
      }
    };
#pragma unroll
    for (int j = 0; j < NPJ; ++j)
#pragma unroll
      for (int c = 0; c < 3; ++c) {
        const uint64_t dv = f2::fma(T[j].h[c], f2::splat(-1.f), B[j].h[c]);   // h1 - h0
        const uint64_t v = f2::fma(ly, dv, T[j].h[c]);                        // fmaf(ly, h1 - h0, h0)
        const uint64_t q = FOLD ? f2::add(v, f2::splat(kBias))                 // 2^23 + rint(v)
                                : rint_biased(v);                              // 1.5 * 2^23 + rint(v)
#pragma unroll
        for (int d = 0; d < ND; ++d)
          if (d == 0 || d < nd) put(dl[d].o[c], dl[d].a[c], dl[d].b[c], j, q);
      }
#pragma unroll
    for (int d = 0; d < ND; ++d)
#pragma unroll
      for (int c = 0; c < 3; ++c) dl[d].o[c] += dl[d].rstride;
  };

  pw::group_sync(fr);                           // row table, mbarrier init visible
  int r = 0;                                        // next output row (warp-uniform)
  uint32_t cy0, cl;                                 // its table entry (y0, lambda bits)
  asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(cy0), "=r"(cl) : "r"(s_tab));
  // every output row whose y0 is `y`, from the lerps of rows y (T) and y + 1 (B)
  auto emit_rows = [&](const Row3 (&T)[NPJ], const Row3 (&B)[NPJ], int y) {
    while ((int)cy0 == y) {
      emit(T, B, __uint_as_float(cl));
      ++r;
      asm volatile("ld.shared.v2.u32 {%0, %1}, [%2];" : "=r"(cy0), "=r"(cl) : "r"(s_tab + 8u * r));
    }
  };

  // 4-pixel groups of a row that any tap reads: [qlo, qlo + nq) (taps i0 in [x_lo, x_hi], i1 = i0 + 1)
  const int qlo = (x_lo - x16) >> 2, nq = ((x_hi + 1 - x16) >> 2) - qlo + 1;
  for (int k = 0; k < nquads; ++k) {
    const int yq = ybase + 4 * k;
    const uint32_t stg = s_stage + (uint32_t)(k % pw::kStages) * stb;
    const uint32_t buf = s_rgb + (uint32_t)(k & 1) * (4u * pw::kRow);
    st::mbar_wait_sleep(s_bar + 8u * (uint32_t)(k % pw::kStages), (uint32_t)(k / pw::kStages) & 1u);
    // conversion: units (UV row u, 4-pixel group q) over the group's 64 lanes; a unit converts
    // the two Y rows sharing UV row u (rows outside the band hold stale bytes: converted, unread)
    const int units = yq + 2 <= y_last ? 2 * nq : nq;  // UV row 1 of the last quad may be unused
    for (int i = gt; i < units; i += 64) {
      const int u = i >= nq ? 1 : 0, q = qlo + i - u * nq;
      const uint32_t uv = st::lds32(stg + (uint32_t)(4 + u) * gw + 4u * q);
      const st::Chroma3 k0 = st::chroma_at<0>(uv, cm), k1 = st::chroma_at<16>(uv, cm);
      const uint32_t yt = st::lds32(stg + (uint32_t)(2 * u) * gw + 4u * q);
      const uint32_t yb = st::lds32(stg + (uint32_t)(2 * u + 1) * gw + 4u * q);
      const uint32_t o = buf + (uint32_t)(2 * u) * pw::kRow + 16u * q;
      st::sts128(o, make_uint4(st::rgbx_dpx(st::byte_of<0>(yt), k0, cm), st::rgbx_dpx(st::byte_of<1>(yt), k0, cm),
                               st::rgbx_dpx(st::byte_of<2>(yt), k1, cm), st::rgbx_dpx(st::byte_of<3>(yt), k1, cm)));
      st::sts128(o + pw::kRow, make_uint4(st::rgbx_dpx(st::byte_of<0>(yb), k0, cm), st::rgbx_dpx(st::byte_of<1>(yb), k0, cm),
                                          st::rgbx_dpx(st::byte_of<2>(yb), k1, cm), st::rgbx_dpx(st::byte_of<3>(yb), k1, cm)));
    }
    // one group barrier per quad: quad k converted (buffer k & 1), its stage drained, and the
    // walk of quad k - 1 (buffer (k + 1) & 1, rewritten by quad k + 1) finished in both warps
    pw::group_sync(fr);
    if (half == (k & 1) && k + pw::kStages < nquads) {   // the two warps take turns
      if (lane < 6) asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      stage(k + pw::kStages);
    }
    if (yq >= y_first) {
      hrows(X, 0u);
      emit_rows(Yr, X, yq - 1);
    }
    if (yq + 1 <= y_last) {
      hrows(Yr, (uint32_t)pw::kRow);
      emit_rows(X, Yr, yq);
    }
    if (yq + 2 <= y_last) {
      hrows(X, 2u * pw::kRow);
      emit_rows(Yr, X, yq + 1);
    }
    if (yq + 3 <= y_last) {
      hrows(Yr, 3u * pw::kRow);
      emit_rows(X, Yr, yq + 2);
    }
    const uint32_t flipb = (k & 1) ? 0u - 4u * pw::kRow : 4u * pw::kRow;   // next quad's buffer
#pragma unroll
    for (int j = 0; j < NPJ; ++j) {
      ca[j] += flipb;
      cb[j] += flipb;
    }
  }
  // rows at the bottom clamp (y0 == y1 == y_last, lambda 0): emitted from H(y_last) twice
  if (y_last & 1) emit_rows(Yr, Yr, y_last);
  else emit_rows(X, X, y_last);
}

}  // namespace sand
