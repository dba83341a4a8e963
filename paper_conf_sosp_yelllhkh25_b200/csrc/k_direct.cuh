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

// NV12 pixel x of a row pair (Y row, UV row) as an RGBx word
__device__ __forceinline__ uint32_t pixel(const uint8_t* __restrict__ yrow, const uint8_t* __restrict__ uvrow, int x) {
  const uint32_t Y = __ldg(yrow + x);
  const uint32_t uv = __ldg(reinterpret_cast<const uint16_t*>(uvrow + (x & ~1)));
  return st::rgbx_dpx(Y, st::chroma_at<0>(uv));
}

// horizontal lerps of source row y at the thread's four taps (R#12)
__device__ __forceinline__ void hrow(rs::Row3& r, const uint8_t* __restrict__ Yp, const uint8_t* __restrict__ UVp,
                                     uint32_t pitch, int y, int xa0, int xa1, int xb0, int xb1, uint64_t lx) {
  const uint8_t* yrow = Yp + (size_t)y * pitch;
  const uint8_t* uvrow = UVp + (size_t)(y >> 1) * pitch;
  const uint32_t a0 = pixel(yrow, uvrow, xa0), a1 = pixel(yrow, uvrow, xa1);
  const uint32_t b0 = pixel(yrow, uvrow, xb0), b1 = pixel(yrow, uvrow, xb1);
  r.h[0] = rs::hlerp<0>(a0, a1, b0, b1, lx);
  r.h[1] = rs::hlerp<1>(a0, a1, b0, b1, lx);
  r.h[2] = rs::hlerp<2>(a0, a1, b0, b1, lx);
}

// both source rows of an output row at once: the sixteen loads are issued before any
// conversion so their latencies overlap
__device__ __forceinline__ void hrow2(rs::Row3& t, rs::Row3& b, const uint8_t* __restrict__ Yp,
                                      const uint8_t* __restrict__ UVp, uint32_t pitch, int y0, int y1, int xa0,
                                      int xa1, int xb0, int xb1, uint64_t lx) {
  const uint8_t* yr[2] = {Yp + (size_t)y0 * pitch, Yp + (size_t)y1 * pitch};
  const uint8_t* uvr[2] = {UVp + (size_t)(y0 >> 1) * pitch, UVp + (size_t)(y1 >> 1) * pitch};
  const int xs[4] = {xa0, xa1, xb0, xb1};
  uint32_t Y[2][4], UV[2][4];
#pragma unroll
  for (int r = 0; r < 2; ++r)
#pragma unroll
    for (int k = 0; k < 4; ++k) {
      Y[r][k] = __ldg(yr[r] + xs[k]);
      UV[r][k] = __ldg(reinterpret_cast<const uint16_t*>(uvr[r] + (xs[k] & ~1)));
    }
  uint32_t q[2][4];
#pragma unroll
  for (int r = 0; r < 2; ++r)
#pragma unroll
    for (int k = 0; k < 4; ++k) q[r][k] = st::rgbx_dpx(Y[r][k], st::chroma_at<0>(UV[r][k]));
#pragma unroll
  for (int c = 0; c < 3; ++c) {
    t.h[c] = c == 0 ? rs::hlerp<0>(q[0][0], q[0][1], q[0][2], q[0][3], lx)
                    : (c == 1 ? rs::hlerp<1>(q[0][0], q[0][1], q[0][2], q[0][3], lx)
                              : rs::hlerp<2>(q[0][0], q[0][1], q[0][2], q[0][3], lx));
    b.h[c] = c == 0 ? rs::hlerp<0>(q[1][0], q[1][1], q[1][2], q[1][3], lx)
                    : (c == 1 ? rs::hlerp<1>(q[1][0], q[1][1], q[1][2], q[1][3], lx)
                              : rs::hlerp<2>(q[1][0], q[1][1], q[1][2], q[1][3], lx));
  }
}

}  // namespace dg

// One CTA = one work item x one band of RB output rows; thread = output column pair.
template <int DT, bool VEC>
__global__ void __launch_bounds__(128, 5) k_direct(const LaunchParams p, int RB, int nbands) {
  using namespace rs;
  const int item_idx = blockIdx.x / nbands;
  const int band = blockIdx.x - item_idx * nbands;
  const WorkItem w = p.items[item_idx];
  if (w.flags & 1u) return;
  const GroupParams& g = p.groups[w.gp];
  const int Wo = g.out_w, Ho = g.out_h;
  const int oy0 = band * RB;
  if (oy0 >= Ho) return;
  const int nr = min(RB, Ho - oy0);
  const uint8_t* Yp = p.slab + w.y_off;
  const uint8_t* UVp = Yp + (size_t)w.pitch * w.src_h;
  const uint32_t pitch = w.pitch;
  const int nd = (int)w.n_dest;
  const uint32_t* dests = p.dests + w.dest_begin;
  const int pairs = (Wo + 1) >> 1;
  for (int pair = threadIdx.x; pair < pairs; pair += blockDim.x) {
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
    Row3 T, B;              // horizontal lerps of source rows yT (top) and yB (bottom)
    int yT = -1, yB = -1;
    for (int rr = 0; rr < nr; ++rr) {
      int y0, y1;
      float ly;
      tap(g.sc_y, g.off_y, oy0 + rr, g.lim_y, g.org_y, y0, y1, ly);
      if (y0 != yT && y0 != yB && y1 != yB && y1 != y0) {   // both rows new (the usual case)
        dg::hrow2(T, B, Yp, UVp, pitch, y0, y1, xa0, xa1, xb0, xb1, lx);
        yT = y0;
        yB = y1;
      }
      if (y0 != yT) {
        if (y0 == yB) {
          T = B;
        } else {
          dg::hrow(T, Yp, UVp, pitch, y0, xa0, xa1, xb0, xb1, lx);
        }
        yT = y0;
      }
      if (y1 != yB) {
        if (y1 == yT) B = T;
        else dg::hrow(B, Yp, UVp, pitch, y1, xa0, xa1, xb0, xb1, lx);
        yB = y1;
      }
      emit<DT, kInlineDests, VEC>(T, B, ly, dl, dt, p, dests, nd, oy0 + rr, ox, vec, has_b);
    }
  }
}

}  // namespace sand
