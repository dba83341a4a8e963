// k_plain.cuh — multi-frame streaming resample kernel for plain items (no rotation / blur)
// with mild scaling (source step <= 2 rows and columns per output row / column): Kinetics RRC,
// SlowFast short-side crops with real scaling, two-view plain groups, tiny (SURVEY §8(a)
// a4-a7, a10, a11).
//
// A TASK is (run of up to FPC items of ONE (clip slot, spatial group), band of output rows).
// Spatial parameters are per clip and group (R#7), so the FPC frames of a task share every tap,
// table and branch: the CTA holds FPC x NQ threads (NQ = output column quads per row; 4 x 56 =
// 224 for 224-wide outputs, no idle lanes) whose control flow is identical, each frame with its
// own source rows in shared memory. Per band, sub-bands of S output rows are processed as
//   * the NV12 rows a sub-band adds are copied HBM -> shared memory by the TMA engine
//     (cp.async.bulk, one copy per row per frame, completion counted on one mbarrier), issued
//     while the previous sub-band is walked (a4);
//   * they are converted once into a per-frame ring of RGBx rows (R#11, the DPX formulation of
//     k_stream.cuh; a5): warps take (frame, UV row) pairs, lanes take 4-pixel groups;
//   * each thread owns four adjacent output columns of its frame for the whole band, keeps the
//     horizontal lerps of the two current source rows in registers (parity-indexed slots, R#12,
//     a6), mirrored for flip (a7), and emits vertical lerp, rint, normalise and 8-byte (bf16)
//     stores per channel to every destination view of the item (a10, a11).
// Row taps, ring offsets and walker actions come from a per-band table in shared memory (one
// LDS.128 broadcast per row). Every fp32 operation is the R#12/R#17 op sequence with IEEE
// rounding: bit-identical to the oracle. Tasks and the exact shared-memory bounds (span, ring
// and staging rows) are computed on the host from the same fp32 tap rule (view.cpp).
#pragma once

namespace sand {
namespace pl {

struct Shape {        // host-chosen launch shape of one batch's plain items
  int fpc;            // frames (items of one run) per CTA
  int nq;             // threads per frame = output column quads of the widest view
  int S;              // output rows per sub-band
  int rb;             // largest band (rows of the row table)
  int ring;           // ring capacity in source rows (>= rows any sub-band spans)
  int raw_rows;       // staging capacity in rows (Y + UV rows any sub-band adds)
  int gw;             // row capacity in pixels (multiple of 16, >= every item's staged span)
  uint32_t ring_magic;   // floor(2^32 / ring) + 1
};

__host__ __device__ inline size_t frame_bytes(const Shape& s) {
  return (size_t)s.ring * s.gw * 4 + rs::a16((size_t)s.raw_rows * s.gw);
}
__host__ __device__ inline size_t smem_bytes(const Shape& s) {
  return rs::a16((size_t)s.rb * 16) + 16 + (size_t)s.fpc * frame_bytes(s);
}

// task encoding (uint2, built by view.cpp): x = first item (index into the launch's items),
// y = pl_task_y(frames, band rows, first output row) (plan_types.h)

// exact quotient of small non-negative integers r / n via a float reciprocal (r < 2^16, n < 2^8)
__device__ __forceinline__ int small_div(int r, float inv_n) { return (int)(((float)r + 0.5f) * inv_n); }

}  // namespace pl

template <int DT, int ND>
__global__ void __launch_bounds__(224, 2) k_plain(const LaunchParams p, const uint2* __restrict__ tasks, pl::Shape sh) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  using namespace rs;
  const int tid = threadIdx.x, nthr = blockDim.x;
  const int warp = tid >> 5, lane = tid & 31, nwarps = nthr >> 5;
  const uint2 tk = tasks[blockIdx.x];
  const int item0 = (int)tk.x;
  const int nfr = (int)(tk.y & 0xffu), nr = (int)((tk.y >> 8) & 0xfffu), Y0 = (int)(tk.y >> 20);
  const WorkItem w0 = p.items[item0];
  const GroupParams& g = p.groups[w0.gp];
  const int Wo = g.out_w;
  const float sc_x = g.sc_x, sc_y = g.sc_y;
  const int off_x = g.off_x, off_y = g.off_y, org_x = g.org_x, org_y = g.org_y;
  const int lim_x = g.lim_x, lim_y = g.lim_y, flip = g.flip;

  uint32_t s_base = (uint32_t)__cvta_generic_to_shared(smem_raw);
  asm volatile("" : "+r"(s_base));
  const uint32_t s_tab = s_base;                                   // rb x 16 B row table
  const uint32_t s_bar = s_tab + (uint32_t)a16((size_t)sh.rb * 16);
  const uint32_t s_fr = s_bar + 16;                                // frame f at s_fr + f * fbytes
  const uint32_t fbytes = (uint32_t)pl::frame_bytes(sh);
  const uint32_t ring_b = (uint32_t)sh.ring * (uint32_t)sh.gw * 4u;   // raw staging after the ring
  const uint32_t rowbytes = (uint32_t)sh.gw * 4u;                  // ring row stride
  const uint32_t rawpitch = (uint32_t)sh.gw;                       // staging row stride

  // staged column span (monotone taps): [x16, x16 + gwi)
  const int x_lo = tap0(sc_x, off_x, 0, org_x);
  int x_hi, dmy;
  float fl;
  tap(sc_x, off_x, Wo - 1, lim_x, org_x, dmy, x_hi, fl);
  const int x16 = x_lo & ~15;
  const int gwi = ((x_hi + 16) & ~15) - x16;
  const int y_first = tap0(sc_y, off_y, Y0, org_y);
  if (gwi > sh.gw) __trap();                                       // host bound violated (never)

  if (tid == 0) {
    st::mbar_init(s_bar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();

  // sub-band k covers band rows [k S, min((k + 1) S, nr)); it adds source rows
  // (y1(last row of k - 1), y1(last row of k)]
  auto last_src = [&](int k) {
    int a, b;
    float l;
    tap(sc_y, off_y, Y0 + min((k + 1) * sh.S, nr) - 1, lim_y, org_y, a, b, l);
    return b;
  };
  // NV12 rows [ya, yb] (Y) and their UV rows of every frame -> staging, one bulk copy per row
  auto stage = [&](int ya, int yb) {
    const int ny = yb - ya + 1, u0 = ya >> 1, nuv = (yb >> 1) - u0 + 1, per = ny + nuv;
    if (lane == 0) st::mbar_arrive_expect_tx(s_bar, (uint32_t)(nfr * per * gwi));
    const float inv = 1.0f / (float)per;
    for (int c = lane; c < nfr * per; c += 32) {
      const int f = pl::small_div(c, inv), r = c - f * per;
      const WorkItem& w = p.items[item0 + f];
      const uint8_t* src = p.slab + w.y_off + x16 +
                           (r < ny ? (size_t)(ya + r) * w.pitch : (size_t)w.pitch * (w.src_h + u0 + r - ny));
      st::bulk_g2s(s_fr + (uint32_t)f * fbytes + ring_b + (uint32_t)r * rawpitch, src, (uint32_t)gwi, s_bar);
    }
  };
  const int nsub = (nr + sh.S - 1) / sh.S;
  int ya = y_first, yb = last_src(0);
  if (warp == 0) stage(ya, yb);

  // row table: ring byte offsets of (y0, y1), walker action and lambda_y per band row
  for (int r = tid; r < nr; r += nthr) {
    int y0, y1;
    float ly;
    tap(sc_y, off_y, Y0 + r, lim_y, org_y, y0, y1, ly);
    const uint32_t s0 = st::ring_mod((uint32_t)(y0 - y_first), (uint32_t)sh.ring, sh.ring_magic);
    const uint32_t s1 = st::ring_mod((uint32_t)(y1 - y_first), (uint32_t)sh.ring, sh.ring_magic);
    uint32_t act = st::kActTop | st::kActBot;
    if (r > 0) {
      const int yp = tap0(sc_y, off_y, Y0 + r - 1, org_y);
      act = y0 == yp ? 0u : (y0 == yp + 1 ? st::kActFlip | st::kActBot : act);
    }
    if (y1 == y0) {            // bottom clamp: lambda 0, the bottom set is never read
      act &= ~st::kActBot;
      ly = 0.f;
    }
    st::sts128(s_tab + 16u * (uint32_t)r, make_uint4(s0 * rowbytes, s1 * rowbytes, act, __float_as_uint(ly)));
  }

  // walker: frame f, output columns [ox, ox + 4)
  const int f = tid / sh.nq;
  const int qd = tid - f * sh.nq;
  const int ox = 4 * qd;
  int active = (f < nfr && ox < Wo) ? 1 : 0;
  asm volatile("" : "+r"(active));
  const int fa = min(f, nfr - 1);
  const uint32_t ringf = s_fr + (uint32_t)fa * fbytes;
  uint32_t ca0[2], ca1[2], cb0[2], cb1[2];
  uint64_t lx[2];
#pragma unroll
  for (int j = 0; j < 2; ++j) {
    const int oj = min(ox + 2 * j, Wo - 2);
    const int ja = flip ? Wo - 1 - oj : oj;
    const int jb = flip ? Wo - 2 - oj : oj + 1;
    int a0, a1, b0, b1;
    float la, lb;
    tap(sc_x, off_x, ja, lim_x, org_x, a0, a1, la);
    tap(sc_x, off_x, jb, lim_x, org_x, b0, b1, lb);
    ca0[j] = 4u * (uint32_t)(a0 - x16);
    ca1[j] = 4u * (uint32_t)(a1 - x16);
    cb0[j] = 4u * (uint32_t)(b0 - x16);
    cb1[j] = 4u * (uint32_t)(b1 - x16);
    lx[j] = f2::pack(__float_as_uint(la), __float_as_uint(lb));
  }
  const WorkItem wf = p.items[item0 + fa];
  const int nd = (int)wf.n_dest;
  const uint32_t* dests = p.dests + wf.dest_begin;
  Dest dl[ND];
#pragma unroll
  for (int d = 0; d < ND; ++d) dl[d] = make_dest(p, dests[d < nd ? d : 0], Y0, ox);
  Row3 X[2], Y[2];
#pragma unroll
  for (int j = 0; j < 2; ++j)
#pragma unroll
    for (int c = 0; c < 3; ++c) X[j].h[c] = Y[j].h[c] = 0ull;
  int top = 0;
  auto hrows = [&](Row3 (&R)[2], uint32_t rowaddr) {
#pragma unroll
    for (int j = 0; j < 2; ++j) st::hrow_s(R[j], rowaddr, ca0[j], ca1[j], cb0[j], cb1[j], lx[j]);
  };

  uint32_t phase = 0;
  bool staged = true;
  for (int k = 0; k < nsub; ++k) {
    if (staged) {
      st::mbar_wait(s_bar, phase);
      phase ^= 1u;
    }
    __syncthreads();                       // walk(k - 1) done: its ring rows may be overwritten
    if (staged) {                          // convert rows [ya, yb] of every frame into the rings
      const int ny = yb - ya + 1, u0 = ya >> 1, nuv = (yb >> 1) - u0 + 1;
      const int q4 = gwi >> 2;
      const float inv = 1.0f / (float)nuv;
      for (int rr = warp; rr < nfr * nuv; rr += nwarps) {
        const int fr = pl::small_div(rr, inv), u = rr - fr * nuv;
        const uint32_t fbase = s_fr + (uint32_t)fr * fbytes;
        const uint32_t raw = fbase + ring_b;
        const int yt = 2 * (u0 + u);
        const bool ptop = yt >= ya, pbot = yt + 1 <= yb;
        const uint32_t st_ = st::ring_mod((uint32_t)(yt - y_first + sh.ring), (uint32_t)sh.ring, sh.ring_magic);
        const uint32_t sb_ = st_ + 1 == (uint32_t)sh.ring ? 0u : st_ + 1;
        const uint32_t yrow_t = raw + (uint32_t)(yt - ya) * rawpitch;
        const uint32_t uvrow = raw + (uint32_t)(ny + u) * rawpitch;
        const uint32_t out_t = fbase + st_ * rowbytes, out_b = fbase + sb_ * rowbytes;
        for (int q = lane; q < q4; q += 32) {
          const uint32_t uv = st::lds32(uvrow + 4u * q);
          const st::Chroma3 c0 = st::chroma_at<0>(uv), c1 = st::chroma_at<16>(uv);
          if (ptop) {
            const uint32_t yw = st::lds32(yrow_t + 4u * q);
            st::sts128(out_t + 16u * q, make_uint4(st::rgbx_dpx(st::byte_of<0>(yw), c0), st::rgbx_dpx(st::byte_of<1>(yw), c0),
                                                   st::rgbx_dpx(st::byte_of<2>(yw), c1), st::rgbx_dpx(st::byte_of<3>(yw), c1)));
          }
          if (pbot) {
            const uint32_t yw = st::lds32(yrow_t + rawpitch + 4u * q);
            st::sts128(out_b + 16u * q, make_uint4(st::rgbx_dpx(st::byte_of<0>(yw), c0), st::rgbx_dpx(st::byte_of<1>(yw), c0),
                                                   st::rgbx_dpx(st::byte_of<2>(yw), c1), st::rgbx_dpx(st::byte_of<3>(yw), c1)));
          }
        }
      }
    }
    staged = false;
    __syncthreads();                       // rings hold every row of sub-band k; staging drained
    if (k + 1 < nsub) {                    // stage the next sub-band's new rows
      const int na = yb + 1, nb = last_src(k + 1);
      if (nb >= na) {
        if (warp == 0) {
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          stage(na, nb);
        }
        staged = true;
      }
      ya = na;
      yb = max(nb, yb);
    }
    const int r_lo = k * sh.S, r_hi = min(r_lo + sh.S, nr);
    for (int rr = r_lo; rr < r_hi; ++rr) {
      const uint4 rt = st::lds128(s_tab + 16u * (uint32_t)rr);
      const uint32_t act = rt.z;
      const float l = __uint_as_float(rt.w);
      top ^= (act & st::kActFlip) ? 1 : 0;
      if (top == 0) {
        if (act & st::kActTop) hrows(X, ringf + rt.x);
        if (act & st::kActBot) hrows(Y, ringf + rt.y);
        if (active) st::emit_np<DT, ND, 2>(X, Y, l, dl, p, dests, nd, Y0 + rr, ox);
      } else {
        if (act & st::kActTop) hrows(Y, ringf + rt.x);
        if (act & st::kActBot) hrows(X, ringf + rt.y);
        if (active) st::emit_np<DT, ND, 2>(Y, X, l, dl, p, dests, nd, Y0 + rr, ox);
      }
    }
  }
}

}  // namespace sand
