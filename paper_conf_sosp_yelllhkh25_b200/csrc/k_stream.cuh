// k_stream.cuh — streaming resample kernel for mild scaling (source step <= 2 rows/cols per
// output row/col: Kinetics RRC, SlowFast short-side crops).
//
// One CTA = one work item (clip slot, source frame, group) x one super-band of SB output
// rows, processed as sub-bands of S rows:
//   * the NV12 rows a sub-band adds are copied HBM -> shared memory with cp.async one
//     sub-band ahead (double-buffered raw staging, all 16 B requests in flight; a4);
//   * they are converted once to RGBx words in a shared-memory ring of source rows, a
//     thread taking one chroma sample's 2x(4) luma pixels (a5, Q1);
//   * each thread owns an output column pair for the whole super-band and keeps the
//     horizontal lerps of the current two source rows in registers across sub-bands (a6),
//     mirrored for flip (a7); vertical lerp, rint, normalise and the 4-byte stores to every
//     destination view follow (a10, a11).
// Per-CTA setup (tap tables, destination pointers) is amortised over SB rows and no source
// row is converted twice inside a super-band. Arithmetic is the R#12/R#17 op sequence with
// IEEE rounding at each step: bit-identical to the oracle.
#pragma once

namespace sand {
namespace st {

using rs::a16;

struct Shape {      // host-chosen launch shape
  int SB;           // output rows per CTA
  int nsb;          // super-bands per item (ceil(maxHo / SB))
  int S;            // output rows per sub-band
  int ring;         // ring capacity in source rows (<= 255)
  int raw_rows;     // raw staging capacity in rows (Y + UV) per buffer
  int gw;           // max row width in bytes of Y (= words of RGBx), multiple of 16
};

__host__ __device__ inline size_t smem_bytes(const Shape& s, int maxWo) {
  return a16((size_t)maxWo * 8) + a16((size_t)s.SB * 8) + (size_t)s.ring * s.gw * 4 +
         2 * a16((size_t)s.raw_rows * s.gw);
}

__device__ __forceinline__ void stage_rows(uint8_t* raw, const uint8_t* Yp, const uint8_t* UVp, uint32_t pitch,
                                           int x16, int gw, int ya, int yb, int tid, int nthr) {
  // Y rows [ya, yb] then UV rows [ya>>1, yb>>1], each gw bytes from column x16
  const int ny = yb - ya + 1, u0 = ya >> 1, nuv = (yb >> 1) - u0 + 1;
  const int chunks = gw >> 4, total = (ny + nuv) * chunks;
  for (int e = tid; e < total; e += nthr) {
    const int r = e / chunks, k = e - r * chunks;    // once per 16 B request, off the hot loop
    const uint8_t* src = r < ny ? Yp + (size_t)(ya + r) * pitch : UVp + (size_t)(u0 + r - ny) * pitch;
    rs::cp_async16(raw + (size_t)r * gw + k * 16, src + x16 + k * 16);
  }
  asm volatile("cp.async.commit_group;\n" ::: "memory");
}

// convert staged rows [ya, yb] into ring slots (y - y_first) % ring
__device__ __forceinline__ void convert_rows(uint32_t* ring, const uint8_t* raw, int gw, int ya, int yb, int y_first,
                                             int ring_rows, int tid, int nthr) {
  const int ny = yb - ya + 1, u0 = ya >> 1, nuv = (yb >> 1) - u0 + 1;
  const uint8_t* rawUV = raw + (size_t)ny * gw;
  const int q4 = gw >> 2;                       // 4-pixel groups per row
  for (int e = tid; e < nuv * q4; e += nthr) {
    const int u = e / q4, q = e - u * q4;
    const uint32_t uv = *reinterpret_cast<const uint32_t*>(rawUV + (size_t)u * gw + 4 * q);
    const rs::Chroma c0 = rs::chroma(uv & 0xffffu), c1 = rs::chroma(uv >> 16);
    const int yt = 2 * (u0 + u);
#pragma unroll
    for (int h = 0; h < 2; ++h) {
      const int y = yt + h;
      if (y < ya || y > yb) continue;
      const uint32_t yw = *reinterpret_cast<const uint32_t*>(raw + (size_t)(y - ya) * gw + 4 * q);
      int slot = y - y_first;
      slot = slot >= ring_rows ? slot % ring_rows : slot;
      uint4 o;
      o.x = rs::rgbx((int)(yw & 0xffu), c0);
      o.y = rs::rgbx((int)((yw >> 8) & 0xffu), c0);
      o.z = rs::rgbx((int)((yw >> 16) & 0xffu), c1);
      o.w = rs::rgbx((int)(yw >> 24), c1);
      *reinterpret_cast<uint4*>(ring + (size_t)slot * gw + 4 * q) = o;
    }
  }
}

}  // namespace st

template <int DT, bool VEC>
__global__ void __launch_bounds__(256, 3) k_stream(const LaunchParams p, st::Shape sh, int maxWo) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  using namespace rs;
  const int item_idx = blockIdx.x / sh.nsb;
  const int sb = blockIdx.x - item_idx * sh.nsb;
  const WorkItem w = p.items[item_idx];
  if (w.flags & 1u) return;
  const GroupParams& g = p.groups[w.gp];
  const int Wo = g.out_w, Ho = g.out_h;
  const int Y0 = sb * sh.SB;
  if (Y0 >= Ho) return;
  const int nr = min(sh.SB, Ho - Y0);
  const int tid = threadIdx.x, nthr = blockDim.x;

  uint8_t* sp = smem_raw;
  uint2* ctab = reinterpret_cast<uint2*>(sp); sp += a16((size_t)maxWo * 8);
  uint2* rtab = reinterpret_cast<uint2*>(sp); sp += a16((size_t)sh.SB * 8);
  uint32_t* ring = reinterpret_cast<uint32_t*>(sp); sp += (size_t)sh.ring * sh.gw * 4;
  const size_t rawcap = a16((size_t)sh.raw_rows * sh.gw);
  uint8_t* const rawbase = sp;   // two raw staging buffers of rawcap bytes

  // footprint of the super-band (monotone taps)
  const int x_lo = tap0(g.sc_x, g.off_x, 0, g.org_x);
  int x_hi, dmy;
  float fl;
  tap(g.sc_x, g.off_x, Wo - 1, g.lim_x, g.org_x, dmy, x_hi, fl);
  const int x16 = x_lo & ~15;
  const int gw = ((x_hi + 16) & ~15) - x16;
  const int y_first = tap0(g.sc_y, g.off_y, Y0, g.org_y);
  const uint8_t* Yp = p.slab + w.y_off;
  const uint8_t* UVp = Yp + (size_t)w.pitch * w.src_h;

  // sub-band k covers output rows [k*S, min((k+1)*S, nr)); its new source rows are
  // (last row of sub-band k-1, y1(last row of k)]
  auto last_src = [&](int k) {
    int a, b;
    float l;
    tap(g.sc_y, g.off_y, Y0 + min((k + 1) * sh.S, nr) - 1, g.lim_y, g.org_y, a, b, l);
    return b;
  };
  const int nsub = (nr + sh.S - 1) / sh.S;
  int ya = y_first, yb = last_src(0);
  st::stage_rows(rawbase, Yp, UVp, w.pitch, x16, gw, ya, yb, tid, nthr);

  // tap tables (overlap the first copy)
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
    const uint32_t s0 = (uint32_t)((y0 - y_first) % sh.ring), s1 = (uint32_t)((y1 - y_first) % sh.ring);
    rtab[r] = make_uint2(s0 | (s1 << 8) | ((uint32_t)y0 << 16), __float_as_uint(ly));
  }

  // per-thread walker state: output column pair `pair`, kept for the whole super-band
  const int pairs = (Wo + 1) >> 1;
  const bool walker = tid < pairs;
  const int ox = 2 * tid;
  const bool has_b = ox + 1 < Wo;
  const bool vec = has_b && !(Wo & 1);
  uint32_t ca = 0, cb = 0;
  float2 lx = make_float2(0.f, 0.f);
  const int nd = (int)w.n_dest;
  const uint32_t* dests = p.dests + w.dest_begin;
  Dest dl[kInlineDests];
  int dt[kInlineDests];
  int have0 = -1, have1 = -1;
  Row3 S0, S1;

  for (int k = 0; k < nsub; ++k) {
    asm volatile("cp.async.wait_group 0;\n" ::: "memory");
    __syncthreads();                                 // raw[k&1] landed; walk(k-1) finished
    st::convert_rows(ring, rawbase + (size_t)(k & 1) * rawcap, gw, ya, yb, y_first, sh.ring, tid, nthr);
    if (k + 1 < nsub) {                              // stage the next sub-band's new rows
      const int na = yb + 1, nb = last_src(k + 1);
      if (nb >= na) st::stage_rows(rawbase + (size_t)((k + 1) & 1) * rawcap, Yp, UVp, w.pitch, x16, gw, na, nb, tid, nthr);
      ya = na;
      yb = max(nb, yb);
    }
    __syncthreads();                                 // ring holds every row of sub-band k
    if (k == 0 && walker) {                          // tables are visible now
      const int ja = g.flip ? Wo - 1 - ox : ox;
      const int jb = has_b ? (g.flip ? Wo - 2 - ox : ox + 1) : ja;
      const uint2 ta = ctab[ja], tb = ctab[jb];
      ca = ta.x;
      cb = tb.x;
      lx = make_float2(__uint_as_float(ta.y), __uint_as_float(tb.y));
#pragma unroll
      for (int d = 0; d < kInlineDests; ++d)
        if (d < nd) {
          dl[d] = make_dest(p, dests[d], Y0, ox);
          dt[d] = DT >= 0 ? DT : p.views[dests[d] >> 24].dtype;
        }
    }
    if (walker) {
      const int r_lo = k * sh.S, r_hi = min(r_lo + sh.S, nr);
      for (int rr = r_lo; rr < r_hi; ++rr) {
        const uint2 rt = rtab[rr];
        const int s0 = (int)(rt.x & 0xffu), s1 = (int)((rt.x >> 8) & 0xffu), y0 = (int)(rt.x >> 16);
        const float l = __uint_as_float(rt.y);
        const int oy = Y0 + rr;
        // parity slots: rows y0 and y0+1 are held in different registers sets (R#12 taps)
        if (y0 & 1) {
          if (have1 != y0) { hrow(S1, ring + (size_t)s0 * gw, ca, cb, lx); have1 = y0; }
          if (s1 != s0) {
            if (have0 != y0 + 1) { hrow(S0, ring + (size_t)s1 * gw, ca, cb, lx); have0 = y0 + 1; }
            emit<DT, kInlineDests, VEC>(S1, S0, l, dl, dt, p, dests, nd, oy, ox, vec, has_b);
          } else {
            emit<DT, kInlineDests, VEC>(S1, S1, l, dl, dt, p, dests, nd, oy, ox, vec, has_b);
          }
        } else {
          if (have0 != y0) { hrow(S0, ring + (size_t)s0 * gw, ca, cb, lx); have0 = y0; }
          if (s1 != s0) {
            if (have1 != y0 + 1) { hrow(S1, ring + (size_t)s1 * gw, ca, cb, lx); have1 = y0 + 1; }
            emit<DT, kInlineDests, VEC>(S0, S1, l, dl, dt, p, dests, nd, oy, ox, vec, has_b);
          } else {
            emit<DT, kInlineDests, VEC>(S0, S0, l, dl, dt, p, dests, nd, oy, ox, vec, has_b);
          }
        }
      }
    }
  }
}

}  // namespace sand
