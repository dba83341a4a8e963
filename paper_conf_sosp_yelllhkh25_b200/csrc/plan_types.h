// plan_types.h — device-visible materialisation plan (host planner -> CUDA kernels).
//
// A batch (epoch, rank, iteration) is a list of WORK ITEMS. A work item is one
// (clip slot b, source frame f, spatial group q) triple: the source frame is read
// once and every (view, t) of group q that selected frame f is written from it
// (multi-view fan-out; node merging). Items of
// the same (b, f) are adjacent so the groups of one frame share its lines in L2.
#pragma once
#include <stdint.h>
#include <vector_types.h>   // uint2 (LaunchParams::tasks)

#if defined(__CUDACC__)
#define SAND_HD __host__ __device__
#else
#define SAND_HD
#endif

namespace sand {

constexpr int kMaxViews = 8;
constexpr int kMaxGroups = 8;
constexpr int kMaxT = 64;
constexpr int kMaxTaps = 23;  // blur taps (k <= 23)

// Geometry + augmentation of one (clip slot, group). Source coordinate of output
// column ox (after the flip mirror ox' = flip ? Wo-1-ox : ox):
//   s = max(sc_x * ((float)(off_x + ox') + 0.5f) - 0.5f, 0);  i0 = (int)s;
//   i1 = min(i0 + 1, lim_x - 1);  taps at org_x + i0, org_x + i1      (R#12)
// RRC: org = crop origin, off = 0, lim = crop size, sc = (float)w / Wo.
// SHORTSIDE_CROP: org = 0, off = crop offset in the resized frame, lim = frame size,
// sc = (float)W / W'.
struct alignas(16) GroupParams {
  int32_t org_x, org_y, off_x, off_y;
  int32_t lim_x, lim_y, out_w, out_h;
  float sc_x, sc_y, rot_c, rot_s;
  int32_t flip, rot_on, blur_on, blur_r;
  float blur_w[24];
  // colour jitter (R#30): gate, order 0..5, per op (brightness, contrast, saturation) the factor
  // f as float and (float)(1 - f) (computed in double)
  int32_t jit_on, jit_order, pad0, pad1;
  float jit_f[4], jit_a[4];
};

struct alignas(16) WorkItem {
  uint64_t y_off;        // byte offset of the source frame's Y plane in the slab
  uint32_t pitch;        // row pitch of Y and UV planes (UV plane at y_off + pitch*src_h)
  uint32_t src_w, src_h;
  uint32_t gp;           // GroupParams index (absolute within the epoch plan)
  uint32_t dest_begin;   // first destination (absolute within the epoch plan)
  uint32_t n_dest;
  uint32_t clip_slot;    // b
  uint32_t group;        // q
  uint32_t flags;        // bit0: needs the stencil path (rotation or blur)
  uint32_t pad;
};

// One crop of a cached resized frame (object reuse, f2; k_crop.cuh, objcache.cpp)
struct alignas(16) CropItem {
  uint64_t obj;          // byte offset of the object (plane R) in the object slab
  uint32_t obj_w, obj_h; // W', H' (plane pitch W', planes W' * H' bytes apart)
  uint32_t x_off, y_off, flip;
  uint32_t out_w, out_h;
  uint32_t dest_begin, n_dest;
  uint32_t pad;
};

// destination packing: view (8 bits) << 24 | t (8 bits) << 16 | b (16 bits)
SAND_HD inline uint32_t pack_dest(uint32_t view, uint32_t t, uint32_t b) {
  return (view << 24) | (t << 16) | b;
}

struct ViewConst {
  float a[3], b[3];      // y = fmaf(q, a_c, b_c)  (R#17)
  int32_t dtype;         // SAND_U8 / SAND_BF16 / SAND_F32
  int32_t T, out_h, out_w;
  // b'_c = b_c - 2^23 a_c when exactly representable for every channel (fold = 1): then
  // fmaf(2^23 + q, a_c, b'_c) == fmaf(q, a_c, b_c) exactly (the real values are equal and fmaf
  // rounds once), so the kernels normalise the biased rint result without un-biasing it
  float bf[3];
  int32_t fold;
};

// Per-batch launch shape of the direct (no rotation/blur) items, from the plan.
struct BatchShape {
  int32_t has_direct, has_stencil;
  int32_t max_wo, max_ho;
  int32_t cols_bound;     // upper bound of distinct tapped source columns of any item
  float max_scy;          // largest vertical source step (rows per output row)
  int32_t dtype;          // output dtype shared by every view, or -1 if mixed
  int32_t even_wo;        // every view's out_w is even
  int32_t wo_mod4;        // every view's out_w is a multiple of 4
  // stencil (rotation/blur) items
  int32_t st_max_wo, st_max_ho, st_cols_bound;
  float st_max_scy;
  uint32_t n_direct;      // items [0, n_direct) of the batch are direct, the rest stencil items
  int32_t direct_identity;  // every mild direct item has sc_x == sc_y == 1 (k_copy applies)
  int32_t src_w_mod4;       // every source width is a multiple of 4
  // item classes (per item, not per batch): direct items [0, n_mild) have a source step <= 2
  // on both axes (k_plain / k_copy), [n_mild, n_direct) heavier down-scaling (k_direct)
  uint32_t n_mild;
  int32_t max_dests;        // largest destination count of a direct item
  int32_t heavy_max_wo, heavy_max_ho;
  // k_plain: the batch's task slice, the widest staged span (pixels) and the longest band
  uint32_t task_first, n_tasks;
  int32_t pl_gw, pl_rb;
  // the tasks are ordered k_plainw-eligible first (staged span <= kPlainwMaxSpan): the first
  // n_tasks_w of them with widest span pl_gw_w; the rest (wider spans) go to k_plain
  uint32_t n_tasks_w;
  int32_t pl_gw_w;
  int32_t fold;             // every view's normalisation folds the rint bias (ViewConst::fold)
  int32_t has_jitter;       // a stencil item applies colour jitter (k_stencil2 only, R#30)
};

// k_plain task granularity (view.cpp builds the tasks, k_plain.cuh consumes them)
#ifndef SAND_PLAIN_RB
#define SAND_PLAIN_RB 64
#endif
constexpr int kPlainRB = SAND_PLAIN_RB;   // output rows per band
#ifndef SAND_PLAIN_RB_TAIL
#define SAND_PLAIN_RB_TAIL 16
#endif
#ifndef SAND_PLAIN_TAIL_FRAC
#define SAND_PLAIN_TAIL_FRAC 0.25
#endif
constexpr int kPlainRBTail = SAND_PLAIN_RB_TAIL;   // band of the tasks that make up the last part of the work
constexpr double kPlainTailFrac = SAND_PLAIN_TAIL_FRAC;

constexpr int kPlainwMaxSpan = 384;   // widest staged span k_plainw takes (k_plainw.cuh kGWMax)

// k_plain task word: frames | band rows << 8 | first output row << 20
SAND_HD inline uint32_t pl_task_y(uint32_t nfr, uint32_t nr, uint32_t y0) { return nfr | (nr << 8) | (y0 << 20); }

// exact fp32 tap of output index o (R#12), the same op sequence as the kernels' tap()
SAND_HD inline void tap_ref(float sc, int off, int o, int lim, int org, int* i0, int* i1, float* lam) {
  float s = sc * ((float)(off + o) + 0.5f) - 0.5f;
  s = s > 0.f ? s : 0.f;
  const int i = (int)s;
  *lam = s - (float)i;
  *i0 = org + i;
  *i1 = org + (i + 1 < lim - 1 ? i + 1 : lim - 1);
}

// YUV -> RGB coefficients in 2^20 fixed point (R#11 BT.601 / R#29 BT.709): yy = max(Y, 16) cy +
// (2^19 - 16 cy); R = sat((yy + vr v) >> 20), G = sat((yy + vg v + ug u) >> 20),
// B = sat((yy + ub u) >> 20), u = U - 128, v = V - 128
struct ColorM {
  int32_t cy, vr, vg, ug, ub;
  int32_t yk;           // 2^19 - 16 cy: yy = max(Y, 16) cy + yk in one IMAD
  int32_t kr, kg, kb;   // -128 x (vr, vg + ug, ub): the chroma terms from the raw U, V bytes
};
SAND_HD inline ColorM color_matrix_of(int32_t cy, int32_t vr, int32_t vg, int32_t ug, int32_t ub) {
  return ColorM{cy, vr, vg, ug, ub, (1 << 19) - 16 * cy, -128 * vr, -128 * (vg + ug), -128 * ub};
}
SAND_HD inline ColorM color_matrix(int32_t m) {
  return m == 1 ? color_matrix_of(1220945, 1879825, -558796, -223607, 2215014)    // BT.709 from Kr, Kb (R#29)
                : color_matrix_of(1220542, 1673527, -852492, -409993, 2116026);  // BT.601, OpenCV (R#11)
}

struct LaunchParams {
  const uint8_t* slab;
  const WorkItem* items;   // this batch's items
  uint32_t n_items;
  const GroupParams* groups;
  const uint32_t* dests;
  void* out[kMaxViews];
  ViewConst views[kMaxViews];
  uint32_t n_views;
  uint32_t batch;          // B
  const uint2* tasks;      // k_plain tasks of this batch (view.cpp)
  ColorM cm;               // the spec's YUV -> RGB matrix (kernel-parameter constants)
};

}  // namespace sand
