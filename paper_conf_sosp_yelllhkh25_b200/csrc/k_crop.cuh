// k_crop.cuh — crops of cached resized frames (R#27).
//
// A cached object is the whole frame resized to W' x H' (uint8 planes R, G, B: Q2 of every crop
// position of a short-side view, R#10/R#12). A crop (x_off, y_off, Wo x Ho) with flip is then
// out[c][oy][ox] = obj[c][y_off + oy][x_off + (flip ? Wo - 1 - ox : ox)], normalised (R#17) and
// stored to every destination view of the item (a7, a10, a11): bit-identical to resampling the
// crop from the NV12 frame, because the short-side map samples output column o at resized
// column off + o with the same fp32 rule. CTA = (crop item, band of kCropRB rows); a thread
// owns four adjacent output columns of a row: 4 bytes per channel from two aligned 32-bit loads
// and a funnel shift at the row's own alignment (W' may be odd; reversed by PRMT under flip), byte -> float by the 2^23 exponent trick,
// packed normalise, 8-byte (bf16) stores.
#pragma once

namespace sand {

// CropItem: plan_types.h

constexpr int kCropRB = 32;   // output rows per CTA

template <int DT>
__global__ void __launch_bounds__(256) k_crop(const LaunchParams p, const uint8_t* __restrict__ slab,
                                              const CropItem* __restrict__ items, int nbands) {
  using namespace rs;
  const int item_idx = blockIdx.x / nbands, band = blockIdx.x - item_idx * nbands;
  const CropItem it = items[item_idx];
  const int Wo = (int)it.out_w, Ho = (int)it.out_h;
  const int quads = Wo >> 2;
  const int rpi = (int)blockDim.x / quads;              // rows per CTA pass
  const int r0 = (int)threadIdx.x / quads;
  if (r0 >= rpi) return;
  const int qd = (int)threadIdx.x - r0 * quads;
  const int ox = 4 * qd;
  const int y_begin = band * kCropRB, y_end = min(Ho, y_begin + kCropRB);
  // first of the 4 source columns (contiguous; reversed under flip)
  const int sx = (int)it.x_off + (it.flip ? Wo - 4 - ox : ox);
  const size_t plane = (size_t)it.obj_w * it.obj_h;
  const uint8_t* base = slab + it.obj + (size_t)it.y_off * it.obj_w + sx;
  const uint32_t* dests = p.dests + it.dest_begin;
  const int nd = (int)it.n_dest;
  for (int oy = y_begin + r0; oy < y_end; oy += rpi) {
    uint32_t w[3];
#pragma unroll
    for (int c = 0; c < 3; ++c) {
      // 4 bytes at any alignment (W' may be odd): two aligned words and a funnel shift
      const uintptr_t a = reinterpret_cast<uintptr_t>(base + (size_t)c * plane + (size_t)oy * it.obj_w);
      const uint32_t* al = reinterpret_cast<const uint32_t*>(a & ~(uintptr_t)3);
      const uint32_t sh = 8u * (uint32_t)(a & 3);
      const uint32_t lo = __ldg(al);
      const uint32_t hi = sh ? __ldg(al + 1) : 0u;
      const uint32_t v = __funnelshift_r(lo, hi, sh);               // bytes sx .. sx + 3
      w[c] = it.flip ? __byte_perm(v, 0u, 0x0123) : v;              // output order
    }
    for (int d = 0; d < nd; ++d) {
      const Dest e = make_dest(p, dests[d], oy, ox);
#pragma unroll
      for (int c = 0; c < 3; ++c) {
        uint8_t* o = e.row + (size_t)c * e.cstride;
        if constexpr (DT == SAND_U8) {
          *reinterpret_cast<uint32_t*>(o) = w[c];
        } else {
          // q as exact floats: [byte, 0, 0, 0x4B] = 2^23 + q, minus 2^23
          const uint64_t b01 = f2::pack(__byte_perm(w[c], 0x4B000000u, 0x7440), __byte_perm(w[c], 0x4B000000u, 0x7441));
          const uint64_t b23 = f2::pack(__byte_perm(w[c], 0x4B000000u, 0x7442), __byte_perm(w[c], 0x4B000000u, 0x7443));
          const uint64_t q01 = f2::add(b01, f2::splat(-kBias)), q23 = f2::add(b23, f2::splat(-kBias));
          const uint64_t a2 = f2::splat(e.a[c]), bb = f2::splat(e.b[c]);
          const uint64_t y01 = f2::fma(q01, a2, bb), y23 = f2::fma(q23, a2, bb);   // fmaf(q, a_c, b_c)
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
  }
}

}  // namespace sand
