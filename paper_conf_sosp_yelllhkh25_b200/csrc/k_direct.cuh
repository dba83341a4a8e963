// k_direct.cuh — direct-gather resample kernel for heavy down-scaling (source step > 2 rows or
// columns per output row/column: the 1080p Ray trials; SURVEY §8(a) a4-a7, a10, a11;
// DESIGN.md §7).
//
// At a source step above 2, no source pixel feeds two output columns (or two output rows), so
// there is nothing to share through shared memory: each thread owns an output column pair,
// walks down a band of output rows, and for every new source row loads exactly the eight
// NV12 pixels its two columns tap (Y bytes and the UV pairs of their 2x2 chroma blocks,
// read-only path, all loads of a row in flight together), converts them to RGBx words in
// registers (OpenCV integer BT.601, R#11), and runs the same packed fp32 lerp / rint /
// normalise / store sequence as the streaming kernel (R#12, R#17). No shared memory and no
// barriers: occupancy is bounded only by registers, which hides the gather latency.
// Views of one group that selected the same frame are written from the same registers (a11).
#pragma once

namespace sand {
namespace dg {

// One NV12 pixel as three biased floats 2^23 + channel (R#11): the OpenCV integer BT.601
// value sat((yy + term) >> 20) is relu(min(yy + term, 2^28 - 1)) >> 20 (one DPX add-min-relu),
// and the shift plus the 0x4B exponent byte are one IMAD.HI with addend; no byte packing.
struct Px3 {
  uint32_t c[3];
};
__device__ __forceinline__ Px3 px3(uint32_t Y, uint32_t uv, const ColorM& m) {
  const st::Chroma3 k = st::chroma_at<0>(uv, m);
  const int yy = (int)max(Y, 16u) * m.cy + m.yk;
  Px3 p;
  p.c[0] = __umulhi((uint32_t)__viaddmin_s32_relu(yy, k.r, 0x0FFFFFFF), 1u << 12) + 0x4B000000u;
  p.c[1] = __umulhi((uint32_t)__viaddmin_s32_relu(yy, k.g, 0x0FFFFFFF), 1u << 12) + 0x4B000000u;
  p.c[2] = __umulhi((uint32_t)__viaddmin_s32_relu(yy, k.b, 0x0FFFFFFF), 1u << 12) + 0x4B000000u;
  return p;
}

// horizontal lerp of channel values given as biased floats, both columns packed (R#12)
__device__ __forceinline__ uint64_t hlerp_b(uint32_t a0, uint32_t a1, uint32_t b0, uint32_t b1, uint64_t lx) {
  const uint64_t P0 = rs::f2::pack(a0, b0), P1 = rs::f2::pack(a1, b1);
  const uint64_t d = rs::f2::fma(P0, rs::f2::splat(-1.f), P1);     // p1 - p0 (exact)
  return rs::f2::fma(lx, d, rs::f2::add(P0, rs::f2::splat(-rs::kBias)));   // fmaf(l, p1 - p0, p0)
}

// horizontal lerps of the source rows of `nr` (1 or 2) rows at the thread's four taps; all
// loads are issued before any conversion so their latencies overlap
template <int NR>
__device__ __forceinline__ void hrows(rs::Row3* out, const uint8_t* __restrict__ Yp, const uint8_t* __restrict__ UVp,
                                      uint32_t pitch, const int (&ys)[2], int xa0, int xa1, int xb0, int xb1,
                                      uint64_t lx, const ColorM& cm) {
  const int xs[4] = {xa0, xa1, xb0, xb1};
  uint32_t Y[NR][4], UV[NR][4];
#pragma unroll
  for (int r = 0; r < NR; ++r) {
    const uint8_t* yr = Yp + (size_t)ys[r] * pitch;
    const uint8_t* uvr = UVp + (size_t)(ys[r] >> 1) * pitch;
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      Y[r][k] = __ldg(yr + xs[k]);
      UV[r][k] = __ldg(reinterpret_cast<const uint16_t*>(uvr + (xs[k] & ~1)));
    }
  }
#pragma unroll
  for (int r = 0; r < NR; ++r) {
    Px3 q[4];
#pragma unroll
    for (int k = 0; k < 4; ++k) q[k] = px3(Y[r][k], UV[r][k], cm);
#pragma unroll
    for (int c = 0; c < 3; ++c) out[r].h[c] = hlerp_b(q[0].c[c], q[1].c[c], q[2].c[c], q[3].c[c], lx);
  }
}

}  // namespace dg

// One CTA = one work item x one band of RB output rows x one chunk of P column pairs; the
// band is split into two halves and thread t = (half t / P, column pair chunk * P + t % P),
// so P = 112 gives 224 threads (seven full warps) for 224-wide outputs.
#ifndef SAND_DIRECT_PF
#define SAND_DIRECT_PF 1
#endif
#ifndef SAND_DIRECT_MINB
#define SAND_DIRECT_MINB 3
#endif
template <int DT, bool VEC>
__global__ void __launch_bounds__(256, SAND_DIRECT_MINB) k_direct(const LaunchParams p, int RB, int nbands, int nchunks) {
  using namespace rs;
  const int item_idx = blockIdx.x / (nbands * nchunks);
  const int rest = blockIdx.x - item_idx * (nbands * nchunks);
  const int band = rest / nchunks, chunk = rest - band * nchunks;
  const WorkItem w = p.items[item_idx];
  if (w.flags & 1u) return;
  const GroupParams& g = p.groups[w.gp];
  const int Wo = g.out_w, Ho = g.out_h;
  const int pairs = (Wo + 1) >> 1;
  const int P = (int)blockDim.x >> 1;                  // threads per half-band
  const int half = (int)threadIdx.x >= P ? 1 : 0;
  const int pair = chunk * P + (int)threadIdx.x - half * P;
  const int hb = (RB + 1) >> 1;
  const int oy0 = band * RB + half * hb;
  const int band_end = min(Ho, band * RB + RB);
  if (oy0 >= band_end || pair >= pairs) return;
  const int nr = min(hb, band_end - oy0);
  const uint8_t* Yp = p.slab + w.y_off;
  const uint8_t* UVp = Yp + (size_t)w.pitch * w.src_h;
  const uint32_t pitch = w.pitch;
  const int nd = (int)w.n_dest;
  const uint32_t* dests = p.dests + w.dest_begin;
  {
    const int ox = 2 * pair;
    const bool has_b = ox + 1 < Wo;
    const bool vec = has_b && !(Wo & 1);
    const int ja = g.flip ? Wo - 1 - ox : ox;                       // flip mirrors x (a7)
    const int jb = has_b ? (g.flip ? Wo - 2 - ox : ox + 1) : ja;
    int xa0, xa1, xb0, xb1;
    float la, lb;
    tap(g.sc_x, g.off_x, ja, g.lim_x, g.org_x, xa0, xa1, la);
    tap(g.sc_x, g.off_x, jb, g.lim_x, g.org_x, xb0, xb1, lb);
    const uint64_t lx = f2::pack(la, lb);
    Dest dl[kInlineDests];
    int dt[kInlineDests];
#pragma unroll
    for (int d = 0; d < kInlineDests; ++d)
      if (d < nd) {
        dl[d] = make_dest(p, dests[d], oy0, ox);
        dt[d] = DT >= 0 ? DT : p.views[dests[d] >> 24].dtype;
      }
#if SAND_DIRECT_PF
    // software-pipelined walk: the 16 NV12 loads of output row rr + 1 are in flight while row
    // rr is converted, lerped and stored (both tap rows are reconverted every row, which only
    // repeats work when the vertical step is below 2)
    {
      uint32_t Yc[2][4], UVc[2][4];
      float lyc;
      // unsigned 32-bit column offsets (no sign extension in the 64-bit address arithmetic)
      const uint32_t xs[4] = {(uint32_t)xa0, (uint32_t)xa1, (uint32_t)xb0, (uint32_t)xb1};
      const uint32_t xuv[4] = {xs[0] & ~1u, xs[1] & ~1u, xs[2] & ~1u, xs[3] & ~1u};
      auto load_row = [&](int oy, uint32_t (&Yv)[2][4], uint32_t (&UVv)[2][4], float& ly) {
        int y0, y1;
        tap(g.sc_y, g.off_y, oy, g.lim_y, g.org_y, y0, y1, ly);
        const uint32_t ys[2] = {(uint32_t)y0, (uint32_t)y1};
#pragma unroll
        for (int r = 0; r < 2; ++r) {
          const uint8_t* yr = Yp + (size_t)(ys[r] * pitch);          // frame offsets fit 32 bits
          const uint8_t* uvr = UVp + (size_t)((ys[r] >> 1) * pitch);
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            Yv[r][k] = __ldg(yr + xs[k]);
            UVv[r][k] = __ldg(reinterpret_cast<const uint16_t*>(uvr + xuv[k]));
          }
        }
      };
      load_row(oy0, Yc, UVc, lyc);
      for (int rr = 0; rr < nr; ++rr) {
        uint32_t Yn[2][4], UVn[2][4];
        float lyn = 0.f;
        if (rr + 1 < nr) load_row(oy0 + rr + 1, Yn, UVn, lyn);
        Row3 tb[2];
#pragma unroll
        for (int r = 0; r < 2; ++r) {
          dg::Px3 q[4];
#pragma unroll
          for (int k = 0; k < 4; ++k) q[k] = dg::px3(Yc[r][k], UVc[r][k], p.cm);
#pragma unroll
          for (int c = 0; c < 3; ++c) tb[r].h[c] = dg::hlerp_b(q[0].c[c], q[1].c[c], q[2].c[c], q[3].c[c], lx);
        }
        // y1 == y0 at the bottom edge: both rows are the same row, lerp weight irrelevant
        emit<DT, kInlineDests, VEC>(tb[0], tb[1], lyc, dl, dt, p, dests, nd, oy0 + rr, ox, vec, has_b);
#pragma unroll
        for (int r = 0; r < 2; ++r)
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            Yc[r][k] = Yn[r][k];
            UVc[r][k] = UVn[r][k];
          }
        lyc = lyn;
      }
    }
    return;
#endif
    Row3 T, B;              // horizontal lerps of source rows yT (top) and yB (bottom)
    int yT = -1, yB = -1;
    for (int rr = 0; rr < nr; ++rr) {
      int y0, y1;
      float ly;
      tap(g.sc_y, g.off_y, oy0 + rr, g.lim_y, g.org_y, y0, y1, ly);
      const int ys2[2] = {y0, y1};
      if (y0 != yT && y0 != yB && y1 != yB && y1 != y0) {   // both rows new (the usual case)
        Row3 tb[2];
        dg::hrows<2>(tb, Yp, UVp, pitch, ys2, xa0, xa1, xb0, xb1, lx, p.cm);
        T = tb[0];
        B = tb[1];
        yT = y0;
        yB = y1;
      }
      if (y0 != yT) {
        if (y0 == yB) {
          T = B;
        } else {
          dg::hrows<1>(&T, Yp, UVp, pitch, ys2, xa0, xa1, xb0, xb1, lx, p.cm);
        }
        yT = y0;
      }
      if (y1 != yB) {
        if (y1 == yT) {
          B = T;
        } else {
          const int ys1[2] = {y1, y1};
          dg::hrows<1>(&B, Yp, UVp, pitch, ys1, xa0, xa1, xb0, xb1, lx, p.cm);
        }
        yB = y1;
      }
      emit<DT, kInlineDests, VEC>(T, B, ly, dl, dt, p, dests, nd, oy0 + rr, ox, vec, has_b);
    }
  }
}

}  // namespace sand
