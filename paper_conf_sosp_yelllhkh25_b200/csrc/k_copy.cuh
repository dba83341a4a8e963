// k_copy.cuh — identity-scale items: when a group's
// sample map has sc_x == sc_y == 1 (the SlowFast short side 256 on 256-high sources, R#10), the
// bilinear taps of R#12 are s = off + o exactly, lambda = 0, and fmaf(0, p1 - p0, p0) == p0, so
// Q2 is the converted source pixel itself (bit-identical to the oracle's resample). This
// kernel is the resample with the dead lerps removed: NV12 -> RGB (R#11) -> normalise (R#17)
// -> stores, no shared memory, no barriers.
//
// CTA = (work item, band of RB output rows); thread = 4 adjacent output columns of one row,
// RPI rows per CTA iteration (RPI = blockDim.x / quads). The 4 source Y bytes are contiguous
// (reversed under flip, a7) and come from two aligned 32-bit loads and a funnel shift; their
// chroma samples from two aligned 32-bit UV loads. Requires out_w % 4 == 0 and source widths
// % 4 == 0 (host-checked; every load stays inside the source row).
#pragma once

namespace sand {
namespace cp {

// one NV12 pixel (luma Y, chroma terms k) -> three biased floats 2^23 + channel (R#11), the
// same DPX add-min-relu + IMAD.HI formulation as the other kernels
__device__ __forceinline__ void px(uint32_t Y, const st::Chroma3& k, uint32_t (&c)[3], const ColorM& m) {
  const int yy = (int)max(Y, 16u) * m.cy + m.yk;
  c[0] = __umulhi((uint32_t)__viaddmin_s32_relu(yy, k.r, 0x0FFFFFFF), 1u << 12) + 0x4B000000u;
  c[1] = __umulhi((uint32_t)__viaddmin_s32_relu(yy, k.g, 0x0FFFFFFF), 1u << 12) + 0x4B000000u;
  c[2] = __umulhi((uint32_t)__viaddmin_s32_relu(yy, k.b, 0x0FFFFFFF), 1u << 12) + 0x4B000000u;
}

}  // namespace cp

#ifndef SAND_COPY_UNROLL
#define SAND_COPY_UNROLL 2
#endif
constexpr int kCopyUnroll = SAND_COPY_UNROLL;   // rows in flight per thread (load latency)

// FOLD: the destinations' b fields hold b' = b - 2^23 a (ViewConst::fold): the biased pixel
// 2^23 + q is normalised directly, fmaf(2^23 + q, a, b') == fmaf(q, a, b) exactly
template <int DT, bool FOLD>
__global__ void __launch_bounds__(256) k_copy(const LaunchParams p, int RB, int nbands) {
  using namespace rs;
  const int item_idx = blockIdx.x / nbands;
  const int band = blockIdx.x - item_idx * nbands;
  const WorkItem w = p.items[item_idx];
  const GroupParams& g = p.groups[w.gp];
  const int Wo = g.out_w, Ho = g.out_h;
  const int quads = Wo >> 2;
  const int rpi = (int)blockDim.x / quads;               // rows per CTA iteration
  const int r0 = (int)threadIdx.x / quads;
  if (r0 >= rpi) return;
  const int qd = (int)threadIdx.x - r0 * quads;
  const int ox = 4 * qd;
  const int y_begin = band * RB, y_end = min(Ho, y_begin + RB);
  // source column of output column ox (identity map): org + off + ox', ox' mirrored under flip
  const int sx = g.org_x + g.off_x + (g.flip ? Wo - 4 - ox : ox);   // first of 4 contiguous columns
  const int sy0 = g.org_y + g.off_y;
  const uint8_t* Yp = p.slab + w.y_off;
  const uint8_t* UVp = Yp + (size_t)w.pitch * w.src_h;
  const int ya = sx & ~3, sh = 8 * (sx & 3);
  const int odd = sx & 1;                                 // uniform per item (ox is a multiple of 4)
  const int nd = (int)w.n_dest;
  const uint32_t* dests = p.dests + w.dest_begin;
  // the first two destinations in registers, advanced per row (a third and later: rare)
  Dest dl0 = make_dest(p, dests[0], y_begin + r0, ox, FOLD), dl1 = dl0;
  if (nd > 1) dl1 = make_dest(p, dests[1], y_begin + r0, ox, FOLD);
#pragma unroll (kCopyUnroll)
  for (int oy = y_begin + r0; oy < y_end; oy += rpi) {
    const int sy = sy0 + oy;
    const uint8_t* yrow = Yp + (size_t)sy * w.pitch;
    const uint8_t* uvrow = UVp + (size_t)(sy >> 1) * w.pitch;
    const uint32_t y_lo = __ldg(reinterpret_cast<const uint32_t*>(yrow + ya));
    const uint32_t y_hi = sh ? __ldg(reinterpret_cast<const uint32_t*>(yrow + ya + 4)) : 0u;
    const uint32_t ys = __funnelshift_r(y_lo, y_hi, sh);  // bytes sx .. sx+3
    // chroma samples: pixel sx + j uses the UV pair at byte (sx + j) & ~1 of the UV row
    const int b0 = (sx & ~1) - ya;                        // byte offset of pixel 0's UV pair (0 or 2)
    const uint32_t u_lo = __ldg(reinterpret_cast<const uint32_t*>(uvrow + ya));
    // the second word only when a needed pair reaches it (then it lies inside the row)
    const uint32_t u_hi = (odd || b0) ? __ldg(reinterpret_cast<const uint32_t*>(uvrow + ya + 4)) : 0u;
    const uint64_t uvw = ((uint64_t)u_hi << 32) | u_lo;
    st::Chroma3 k[3];                                     // even sx: 2 samples; odd sx: 3
    k[0] = st::chroma_at<0>((uint32_t)(uvw >> (8 * b0)), p.cm);
    k[1] = st::chroma_at<0>((uint32_t)(uvw >> (8 * b0 + 16)), p.cm);
    if (odd) k[2] = st::chroma_at<0>((uint32_t)(uvw >> (8 * b0 + 32)), p.cm);
    uint32_t c[4][3];                                     // source pixels sx .. sx+3
    if (!odd) {
      cp::px(ys & 0xffu, k[0], c[0], p.cm);
      cp::px((ys >> 8) & 0xffu, k[0], c[1], p.cm);
      cp::px((ys >> 16) & 0xffu, k[1], c[2], p.cm);
      cp::px(ys >> 24, k[1], c[3], p.cm);
    } else {
      cp::px(ys & 0xffu, k[0], c[0], p.cm);
      cp::px((ys >> 8) & 0xffu, k[1], c[1], p.cm);
      cp::px((ys >> 16) & 0xffu, k[1], c[2], p.cm);
      cp::px(ys >> 24, k[2], c[3], p.cm);
    }
    // output column ox + j holds source pixel j (or 3 - j under flip)
    if (g.flip) {                                         // output column ox + j <- source pixel 3 - j
#pragma unroll
      for (int ch = 0; ch < 3; ++ch) {
        uint32_t t = c[0][ch];
        c[0][ch] = c[3][ch];
        c[3][ch] = t;
        t = c[1][ch];
        c[1][ch] = c[2][ch];
        c[2][ch] = t;
      }
    }
    for (int d = 0; d < nd; ++d) {
      const Dest e = d == 0 ? dl0 : (d == 1 ? dl1 : make_dest(p, dests[d], oy, ox, FOLD));
#pragma unroll
      for (int ch = 0; ch < 3; ++ch) {
        const uint32_t t0 = c[0][ch], t1 = c[1][ch], t2 = c[2][ch], t3 = c[3][ch];
        uint8_t* o = e.row + (size_t)ch * e.cstride;
        if constexpr (DT == SAND_U8) {
          *reinterpret_cast<uint32_t*>(o) =
              __byte_perm(__byte_perm(t0, t1, 0x0040), __byte_perm(t2, t3, 0x0040), 0x5410);
        } else {
          const uint64_t a2 = f2::splat(e.a[ch]), b2 = f2::splat(e.b[ch]);
          const uint64_t q01 = FOLD ? f2::pack(t0, t1) : f2::add(f2::pack(t0, t1), f2::splat(-kBias));   // (2^23 +) q
          const uint64_t q23 = FOLD ? f2::pack(t2, t3) : f2::add(f2::pack(t2, t3), f2::splat(-kBias));
          const uint64_t y01 = f2::fma(q01, a2, b2), y23 = f2::fma(q23, a2, b2);   // fmaf(q, a_c, b_c)
          if constexpr (DT == SAND_BF16) {
            const __nv_bfloat162 v0 = __floats2bfloat162_rn(f2::lof(y01), f2::hif(y01));
            const __nv_bfloat162 v1 = __floats2bfloat162_rn(f2::lof(y23), f2::hif(y23));
            *reinterpret_cast<uint2*>(o) =
                make_uint2(*reinterpret_cast<const uint32_t*>(&v0), *reinterpret_cast<const uint32_t*>(&v1));
          } else {
            *reinterpret_cast<uint4*>(o) = make_uint4(f2::lo(y01), f2::hi(y01), f2::lo(y23), f2::hi(y23));
          }
        }
      }
    }
    dl0.row += (size_t)dl0.rstride * rpi;
    dl1.row += (size_t)dl1.rstride * rpi;
  }
}

}  // namespace sand
