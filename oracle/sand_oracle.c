/*
 * sand_oracle.c — CPU ORACLE for SAND's per-batch view materialisation path.
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and bench.py's
 * cpu_baseline / --impl reference legs may load or call this file's library.
 * The product (paper_conf_sosp_yelllhkh25_b200/) never includes, links or calls
 * it, and this file includes nothing from the product.
 *
 * Plain, slow, single-threaded, step-by-step. Each function cites the passage it
 * follows: "P:Lnnn" is /root/reference/PAPER.md line nnn; "R#n" is reading n of
 * DESIGN.md §2 (the table of readings where the paper is silent; it restates
 * SURVEY.md §8(c)). Precision (DESIGN.md §2 R#12/R#20): parameter math (RRC
 * area/ratio, rotation angle, blur weights, normalisation constants) is done in
 * double and cast to float once; pixel math is fp32 with every operation an IEEE
 * correctly-rounded basic op or fmaf, because each stage ends in a uint8
 * quantisation (frames and augmented frames are uint8) and "where
 * floating point decides an integer, both sides take that decision in the same
 * precision". Compile with -O2 -ffp-contract=off (no contraction, no fast-math).
 *
 * Pins (tests/test_oracle_*.py): Philox against Random123 known-answer vectors;
 * partition against torch DistributedSampler; RRC against torchvision's own
 * get_params fed the same uniforms; NV12->RGB against cv2 (exhaustive); resample
 * against torch F.interpolate; flip against torch.flip; rotation against
 * torchvision F.rotate; blur against scipy.ndimage and torchvision; normalise
 * against torchvision normalize; plus invariants and brute force. The temporal
 * pool / shared-window coordination is pinned by invariants only.
 */
#include <math.h>
#include <stddef.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

#define OR_MAX_VIEWS 8
#define OR_MAX_GROUPS 8
#define OR_MAX_T 64

enum { OR_U8 = 0, OR_BF16 = 1, OR_F32 = 2 };
enum { OR_GEOM_RRC = 0, OR_GEOM_SHORTSIDE_CROP = 1 };
enum { OR_PERM = 1, OR_TEMPORAL = 2, OR_RRC = 3, OR_AUG = 4, OR_WINDOW = 5 };

/* One view = one task / trial / pathway (P:L180 video handling + P:L182 augmentation). */
typedef struct {
  uint32_t clip_len, stride;       /* T, temporal stride (P:L180 frames_per_video, frame_stride) */
  int32_t pool_offset;             /* -1 random offset in the shared pool, >=0 fixed (R#5) */
  uint32_t spatial_group;          /* views with equal group share spatial draws (R#6) */
  int32_t geom;                    /* OR_GEOM_* */
  double scale_min, scale_max, ratio_min, ratio_max; /* RRC (R#8) */
  uint32_t short_side;             /* SHORTSIDE_CROP S (R#10) */
  uint32_t out_h, out_w;
  double flip_p, rot_p, rot_max_deg, blur_p, sigma_min, sigma_max;
  uint32_t blur_ksize;
  double blur_truncate;
  double mean[3], std[3];
  int32_t out_dtype;               /* OR_U8 / OR_BF16 / OR_F32 */
  int32_t subsample_of;            /* -1: pool view; k: linspace sub-sample of view k (R#26) */
  int32_t color_matrix;            /* 0: BT.601 (R#11), 1: BT.709 (R#29) */
  double jitter_p, brightness, contrast, saturation;   /* colour jitter (R#30) */
} oracle_view;

typedef struct {
  uint64_t seed;
  uint32_t world_size, batch_size, samples_per_video;
  int32_t drop_last;
  uint32_t n_views;
  int32_t shared_window;           /* P:L295 shared window over all RRC groups */
  uint32_t pool_epochs;            /* pool drawn once per chunk of k epochs (R#25) */
  oracle_view views[OR_MAX_VIEWS];
} oracle_spec;

typedef struct { uint32_t video, n_frames, width, height; } oracle_video_info;

typedef struct {
  uint32_t clip, video, sample, pool_start;
  uint32_t frames[OR_MAX_VIEWS][OR_MAX_T];
  int32_t box[OR_MAX_GROUPS][4];   /* RRC: x0,y0,w,h ; SHORTSIDE: x_off,y_off,W',H' */
  uint32_t flip[OR_MAX_GROUPS], rot_on[OR_MAX_GROUPS], blur_on[OR_MAX_GROUPS], blur_r[OR_MAX_GROUPS];
  double theta[OR_MAX_GROUPS], sigma[OR_MAX_GROUPS];
  uint32_t jitter_on[OR_MAX_GROUPS], jitter_order[OR_MAX_GROUPS];
  double jitter_f[OR_MAX_GROUPS][3];   /* brightness, contrast, saturation factors */
} oracle_clip_meta;

/* ------------------------------------------------------------------------- */
/* O1. Counter-based RNG: Philox4x32-10 (Salmon et al. SC'11, Random123).     */
/* Randomness must be preserved per task; the generator is R#1.  */
/* ------------------------------------------------------------------------- */
void oracle_philox4x32_10(const uint32_t ctr_in[4], const uint32_t key_in[2], uint32_t out[4]) {
  uint32_t c0 = ctr_in[0], c1 = ctr_in[1], c2 = ctr_in[2], c3 = ctr_in[3];
  uint32_t k0 = key_in[0], k1 = key_in[1];
  for (int round = 0; round < 10; ++round) {
    uint64_t p0 = (uint64_t)0xD2511F53u * (uint64_t)c0;
    uint64_t p1 = (uint64_t)0xCD9E8D57u * (uint64_t)c2;
    uint32_t hi0 = (uint32_t)(p0 >> 32), lo0 = (uint32_t)p0;
    uint32_t hi1 = (uint32_t)(p1 >> 32), lo1 = (uint32_t)p1;
    uint32_t n0 = hi1 ^ c1 ^ k0;
    uint32_t n1 = lo1;
    uint32_t n2 = hi0 ^ c3 ^ k1;
    uint32_t n3 = lo0;
    c0 = n0; c1 = n1; c2 = n2; c3 = n3;
    k0 += 0x9E3779B9u;   /* Weyl key schedule */
    k1 += 0xBB67AE85u;
  }
  out[0] = c0; out[1] = c1; out[2] = c2; out[3] = c3;
}

/* counter = (c0 = draw index, c1 = purpose<<24 | group<<16 | sub, c2 = clip, c3 = epoch) */
static void draw(uint64_t seed, uint32_t purpose, uint32_t group, uint32_t sub, uint32_t c0,
                 uint32_t c2, uint64_t epoch, uint32_t out[4]) {
  uint32_t ctr[4] = {c0, (purpose << 24) | ((group & 0xffu) << 16) | (sub & 0xffffu), c2,
                     (uint32_t)epoch};
  /* R#1: the epoch's high word is XORed into the key's high word (epochs >= 2^32 stay distinct) */
  uint32_t key[2] = {(uint32_t)seed, (uint32_t)(seed >> 32) ^ (uint32_t)(epoch >> 32)};
  oracle_philox4x32_10(ctr, key, out);
}

double oracle_u01(uint32_t x) { return (double)x * (1.0 / 4294967296.0); }

/* integer in [0, n): Lemire multiply-shift without rejection (R#1) */
uint32_t oracle_bounded(uint32_t x, uint32_t n) { return (uint32_t)(((uint64_t)x * (uint64_t)n) >> 32); }

/* Bernoulli(p): x < floor(p * 2^32) */
int oracle_bern(uint32_t x, double p) {
  if (p <= 0.0) return 0;
  if (p >= 1.0) return 1;
  uint64_t thr = (uint64_t)floor(p * 4294967296.0);
  return (uint64_t)x < thr;
}

/* ------------------------------------------------------------------------- */
/* O2. Epoch permutation. "Each video must be processed and used exactly once */
/* per epoch". Fisher-Yates, i = n-1 .. 1 (R#2).             */
/* ------------------------------------------------------------------------- */
void oracle_permutation(uint32_t n, uint64_t seed, uint64_t epoch, uint32_t* perm) {
  for (uint32_t i = 0; i < n; ++i) perm[i] = i;
  for (uint32_t i = n; i-- > 1;) {
    uint32_t x[4];
    draw(seed, OR_PERM, 0, 0, 0, i, epoch, x);
    uint32_t j = oracle_bounded(x[0], i + 1);
    uint32_t t = perm[i];
    perm[i] = perm[j];
    perm[j] = t;
  }
}

/* ------------------------------------------------------------------------- */
/* O3. Rank partition: torch DistributedSampler(shuffle=False) over the       */
/* permuted clip list (north_star "DistributedSampler order"; R#3).           */
/* Writes num_samples entries into out; returns num_samples.                  */
/* ------------------------------------------------------------------------- */
uint32_t oracle_num_samples(uint32_t n, uint32_t world, int drop_last) {
  if (drop_last && (n % world) != 0) {
    if (n < world) return 0;
    return (n - world + world - 1) / world;     /* ceil((n - W) / W) */
  }
  return (n + world - 1) / world;                /* ceil(n / W) */
}

uint32_t oracle_partition(const uint32_t* perm, uint32_t n, uint32_t world, uint32_t rank,
                          int drop_last, uint32_t* out) {
  uint32_t num_samples = oracle_num_samples(n, world, drop_last);
  uint64_t total = (uint64_t)num_samples * world;
  /* padded list: position p < n -> perm[p]; p >= n -> perm[(p - n) % n] (wrap-around) */
  uint32_t k = 0;
  for (uint64_t p = rank; p < total; p += world) {
    uint32_t src = p < n ? (uint32_t)p : (uint32_t)((p - n) % n);
    out[k++] = perm[src];
  }
  return k;
}

/* ------------------------------------------------------------------------- */
/* O4. Temporal sampling through the shared frame pool:             */
/* (1) collect T_k and s_k, (2) grid step g = gcd of strides, (3) random      */
/* selection on that grid up to the maximum clip length. R#4, R#5.           */
/* ------------------------------------------------------------------------- */
static uint32_t gcd_u32(uint32_t a, uint32_t b) {
  while (b) { uint32_t t = a % b; a = b; b = t; }
  return a;
}

/* Position i of linspace(0, n - 1, steps) truncated to an integer, exactly (R#26):
   floor(i * (n - 1) / (steps - 1)). PySlowFast's torch.linspace(...).long() gives the same
   positions except where float32 rounding lands just below an integer. */
uint32_t oracle_linspace_index(uint32_t i, uint32_t steps, uint32_t n) {
  if (steps <= 1) return 0;
  return (uint32_t)(((uint64_t)i * (n - 1)) / (steps - 1));
}

void oracle_temporal(const oracle_spec* spec, uint64_t epoch, uint32_t clip, uint32_t n_frames_video,
                     oracle_clip_meta* meta) {
  /* the pool is built from the views that draw from it (subsample_of < 0) */
  uint32_t g = 0;
  for (uint32_t k = 0; k < spec->n_views; ++k)
    if (spec->views[k].subsample_of < 0) g = gcd_u32(g, spec->views[k].stride);
  uint32_t span[OR_MAX_VIEWS];
  uint32_t L = 0;
  for (uint32_t k = 0; k < spec->n_views; ++k) {
    span[k] = (spec->views[k].clip_len - 1) * (spec->views[k].stride / g) + 1;
    if (spec->views[k].subsample_of < 0 && span[k] > L) L = span[k];
  }
  uint32_t P = (L - 1) * g + 1;                  /* frames covered by the pool */
  uint32_t F = n_frames_video;
  uint32_t x[4];
  /* "videos are decoded once and cached for exactly k epochs before refreshing" --
     the pool start is drawn per chunk floor(epoch / k); offsets below stay per epoch (R#25) */
  uint64_t chunk = spec->pool_epochs > 1 ? epoch / spec->pool_epochs : epoch;
  draw(spec->seed, OR_TEMPORAL, 0, 0, 0, clip, chunk, x);
  uint32_t start = oracle_bounded(x[0], (F > P ? F - P : 0) + 1);
  meta->pool_start = start;
  for (uint32_t k = 0; k < spec->n_views; ++k) {
    uint32_t o;
    if (spec->views[k].subsample_of >= 0) continue;     /* filled below from its parent */
    if (spec->views[k].pool_offset >= 0) {
      o = (uint32_t)spec->views[k].pool_offset;
    } else {
      draw(spec->seed, OR_TEMPORAL, 0, 1 + k, 0, clip, epoch, x);
      o = oracle_bounded(x[0], L - span[k] + 1);
    }
    for (uint32_t t = 0; t < spec->views[k].clip_len; ++t) {
      uint32_t idx = start + (o + t * (spec->views[k].stride / g)) * g;
      meta->frames[k][t] = idx < F - 1 ? idx : F - 1;   /* clamp to the last frame (R#4) */
    }
  }
  /* PySlowFast slow pathway (R#26): the parent's frames at linspace positions */
  for (uint32_t k = 0; k < spec->n_views; ++k) {
    int32_t p = spec->views[k].subsample_of;
    if (p < 0) continue;
    for (uint32_t t = 0; t < spec->views[k].clip_len; ++t)
      meta->frames[k][t] = meta->frames[p][oracle_linspace_index(t, spec->views[k].clip_len, spec->views[p].clip_len)];
  }
}

/* ------------------------------------------------------------------------- */
/* O5. Spatial draws per (clip, group): RandomResizedCrop box (torchvision    */
/* get_params, R#8), short-side crop (R#9/R#10), shared window (P:L295,       */
/* R#18), flip / rotation / blur gates (Fig. 9).    */
/* ------------------------------------------------------------------------- */

/* RRC size search: returns 1 and (w,h,x2,x3 of the accepted attempt) or 0 for fallback */
static int rrc_attempts(const oracle_view* v, uint64_t seed, uint64_t epoch, uint32_t clip,
                        uint32_t group, uint32_t W, uint32_t H, int32_t* w_out, int32_t* h_out,
                        uint32_t* x2_out, uint32_t* x3_out) {
  double area = (double)W * (double)H;
  double log_rmin = log(v->ratio_min);
  double log_rmax = log(v->ratio_max);
  for (uint32_t a = 0; a < 10; ++a) {
    uint32_t x[4];
    draw(seed, OR_RRC, group, 0, a, clip, epoch, x);
    double target_area = area * (v->scale_min + (v->scale_max - v->scale_min) * oracle_u01(x[0]));
    double aspect = exp(log_rmin + (log_rmax - log_rmin) * oracle_u01(x[1]));
    double wd = nearbyint(sqrt(target_area * aspect));   /* Python round(): half-even */
    double hd = nearbyint(sqrt(target_area / aspect));
    if (wd > 0.0 && wd <= (double)W && hd > 0.0 && hd <= (double)H) {
      *w_out = (int32_t)wd;
      *h_out = (int32_t)hd;
      *x2_out = x[2];
      *x3_out = x[3];
      return 1;
    }
  }
  return 0;
}

static void rrc_fallback(const oracle_view* v, uint32_t W, uint32_t H, int32_t* w, int32_t* h) {
  double in_ratio = (double)W / (double)H;
  if (in_ratio < v->ratio_min) {
    *w = (int32_t)W;
    *h = (int32_t)nearbyint((double)W / v->ratio_min);
  } else if (in_ratio > v->ratio_max) {
    *h = (int32_t)H;
    *w = (int32_t)nearbyint((double)H * v->ratio_max);
  } else {
    *w = (int32_t)W;
    *h = (int32_t)H;
  }
}

/* box = (x0, y0, w, h) of torchvision RandomResizedCrop.get_params (returns i=y0, j=x0, h, w) */
void oracle_rrc_box(const oracle_view* v, uint64_t seed, uint64_t epoch, uint32_t clip, uint32_t group,
                    uint32_t W, uint32_t H, int32_t box[4]) {
  int32_t w, h;
  uint32_t x2, x3;
  if (rrc_attempts(v, seed, epoch, clip, group, W, H, &w, &h, &x2, &x3)) {
    box[1] = (int32_t)oracle_bounded(x2, H - (uint32_t)h + 1);   /* i = randint(0, H-h+1) */
    box[0] = (int32_t)oracle_bounded(x3, W - (uint32_t)w + 1);   /* j = randint(0, W-w+1) */
  } else {
    rrc_fallback(v, W, H, &w, &h);                              /* central crop */
    box[1] = ((int32_t)H - h) / 2;
    box[0] = ((int32_t)W - w) / 2;
  }
  box[2] = w;
  box[3] = h;
}

/* short side S then crop out_h x out_w at a uniform offset (PySlowFast floor, torchvision RandomCrop) */
void oracle_shortside_box(const oracle_view* v, uint64_t seed, uint64_t epoch, uint32_t clip,
                          uint32_t group, uint32_t W, uint32_t H, int32_t box[4]) {
  uint32_t S = v->short_side, Wp, Hp;
  if (W <= H) {
    Wp = S;
    Hp = (uint32_t)(((uint64_t)H * S) / W);
  } else {
    Wp = (uint32_t)(((uint64_t)W * S) / H);
    Hp = S;
  }
  uint32_t x[4];
  draw(seed, OR_RRC, group, 0, 0, clip, epoch, x);
  box[1] = (int32_t)oracle_bounded(x[2], Hp - v->out_h + 1);
  box[0] = (int32_t)oracle_bounded(x[3], Wp - v->out_w + 1);
  box[2] = (int32_t)Wp;
  box[3] = (int32_t)Hp;
}

/* the view that defines group q's spatial parameters: the lowest-index view of the group */
static int group_leader(const oracle_spec* spec, uint32_t q) {
  for (uint32_t k = 0; k < spec->n_views; ++k)
    if (spec->views[k].spatial_group == q) return (int)k;
  return -1;
}

void oracle_spatial(const oracle_spec* spec, uint64_t epoch, uint32_t clip, uint32_t W, uint32_t H,
                    oracle_clip_meta* meta) {
  uint64_t seed = spec->seed;
  if (spec->shared_window) {
    /* P:L295 (1) sizes of every group's crop, (2) one random window holding the largest,
       (3) each group picks its sub-region inside the window (R#18). */
    int32_t ws[OR_MAX_GROUPS] = {0}, hs[OR_MAX_GROUPS] = {0};
    int32_t Wwin = 0, Hwin = 0;
    for (uint32_t q = 0; q < OR_MAX_GROUPS; ++q) {
      int k = group_leader(spec, q);
      if (k < 0) continue;
      uint32_t x2, x3;
      if (!rrc_attempts(&spec->views[k], seed, epoch, clip, q, W, H, &ws[q], &hs[q], &x2, &x3))
        rrc_fallback(&spec->views[k], W, H, &ws[q], &hs[q]);
      if (ws[q] > Wwin) Wwin = ws[q];
      if (hs[q] > Hwin) Hwin = hs[q];
    }
    uint32_t x[4];
    draw(seed, OR_WINDOW, 0, 0, 0, clip, epoch, x);
    int32_t wy = (int32_t)oracle_bounded(x[0], H - (uint32_t)Hwin + 1);
    int32_t wx = (int32_t)oracle_bounded(x[1], W - (uint32_t)Wwin + 1);
    for (uint32_t q = 0; q < OR_MAX_GROUPS; ++q) {
      if (group_leader(spec, q) < 0) continue;
      draw(seed, OR_WINDOW, q, 1, 0, clip, epoch, x);
      meta->box[q][1] = wy + (int32_t)oracle_bounded(x[0], (uint32_t)(Hwin - hs[q]) + 1);
      meta->box[q][0] = wx + (int32_t)oracle_bounded(x[1], (uint32_t)(Wwin - ws[q]) + 1);
      meta->box[q][2] = ws[q];
      meta->box[q][3] = hs[q];
    }
  } else {
    for (uint32_t q = 0; q < OR_MAX_GROUPS; ++q) {
      int k = group_leader(spec, q);
      if (k < 0) continue;
      if (spec->views[k].geom == OR_GEOM_RRC)
        oracle_rrc_box(&spec->views[k], seed, epoch, clip, q, W, H, meta->box[q]);
      else
        oracle_shortside_box(&spec->views[k], seed, epoch, clip, q, W, H, meta->box[q]);
    }
  }
  /* augmentation gates: flip (Fig. 9), rotation and blur; R#15-R#16 */
  for (uint32_t q = 0; q < OR_MAX_GROUPS; ++q) {
    int k = group_leader(spec, q);
    if (k < 0) continue;
    const oracle_view* v = &spec->views[k];
    uint32_t x[4];
    draw(seed, OR_AUG, q, 0, 0, clip, epoch, x);
    meta->flip[q] = (uint32_t)oracle_bern(x[0], v->flip_p);
    meta->rot_on[q] = (uint32_t)oracle_bern(x[1], v->rot_p);
    meta->theta[q] = (2.0 * oracle_u01(x[2]) - 1.0) * v->rot_max_deg;
    meta->blur_on[q] = (uint32_t)oracle_bern(x[3], v->blur_p);
    draw(seed, OR_AUG, q, 1, 0, clip, epoch, x);
    meta->sigma[q] = v->sigma_min + (v->sigma_max - v->sigma_min) * oracle_u01(x[0]);
    uint32_t rmax = (v->blur_ksize - 1) / 2;
    if (v->blur_truncate <= 0.0) {
      meta->blur_r[q] = rmax;
    } else {
      double rr = floor(v->blur_truncate * meta->sigma[q] + 0.5);
      meta->blur_r[q] = rr < (double)rmax ? (uint32_t)rr : rmax;
    }
    /* colour jitter (R#30): gate, factors U[max(0, 1 - m), 1 + m] (torchvision
       ColorJitter's ranges), then the order of the three ops: one of the 6 permutations of
       (brightness, contrast, saturation) in lexicographic order */
    draw(seed, OR_AUG, q, 2, 0, clip, epoch, x);
    meta->jitter_on[q] = (uint32_t)oracle_bern(x[0], v->jitter_p);
    double mags[3] = {v->brightness, v->contrast, v->saturation};
    for (int i = 0; i < 3; ++i) {
      double lo = mags[i] < 1.0 ? 1.0 - mags[i] : 0.0, hi = 1.0 + mags[i];
      meta->jitter_f[q][i] = lo + (hi - lo) * oracle_u01(x[1 + i]);
    }
    draw(seed, OR_AUG, q, 3, 0, clip, epoch, x);
    meta->jitter_order[q] = oracle_bounded(x[0], 6);
  }
}

/* Plan one clip: video, temporal indices, spatial draws. dataset[k] describes videos[k]. */
void oracle_plan_clip(const oracle_spec* spec, const oracle_video_info* dataset, uint64_t epoch,
                      uint32_t clip, oracle_clip_meta* meta) {
  memset(meta, 0, sizeof(*meta));
  uint32_t S = spec->samples_per_video;
  const oracle_video_info* vi = &dataset[clip / S];
  meta->clip = clip;
  meta->video = vi->video;
  meta->sample = clip % S;
  oracle_temporal(spec, epoch, clip, vi->n_frames, meta);
  oracle_spatial(spec, epoch, clip, vi->width, vi->height, meta);
}

uint64_t oracle_iterations(const oracle_spec* spec, uint32_t n_videos) {
  uint32_t n = n_videos * spec->samples_per_video;
  return oracle_num_samples(n, spec->world_size, spec->drop_last) / spec->batch_size;
}

/* Plan the B clips of (epoch, rank, iteration). Returns 0, or -4 if iteration is out of range. */
int oracle_plan_batch(const oracle_spec* spec, const oracle_video_info* dataset, uint32_t n_videos,
                      uint64_t epoch, uint32_t rank, uint64_t iteration, oracle_clip_meta* metas) {
  uint32_t n = n_videos * spec->samples_per_video;
  if (iteration >= oracle_iterations(spec, n_videos)) return -4;
  uint32_t* perm = (uint32_t*)malloc(sizeof(uint32_t) * (n ? n : 1));
  uint32_t* mine = (uint32_t*)malloc(sizeof(uint32_t) * (n / spec->world_size + 2));
  oracle_permutation(n, spec->seed, epoch, perm);
  oracle_partition(perm, n, spec->world_size, rank, spec->drop_last, mine);
  for (uint32_t b = 0; b < spec->batch_size; ++b)
    oracle_plan_clip(spec, dataset, epoch, mine[iteration * spec->batch_size + b], &metas[b]);
  free(perm);
  free(mine);
  return 0;
}

/* ------------------------------------------------------------------------- */
/* O6. NV12 -> RGB, BT.601 limited range, nearest chroma, OpenCV integer form */
/* (R#11; the paper's op library is OpenCV). Output HWC uint8.        */
/* ------------------------------------------------------------------------- */
static uint8_t sat_u8(int32_t v) { return (uint8_t)(v < 0 ? 0 : (v > 255 ? 255 : v)); }

/* matrix 0: BT.601 limited range, OpenCV's COLOR_YUV2RGB_NV12 integer form (R#11).
   matrix 1: BT.709 limited range (R#29): the same form with coefficients round(c * 2^20) of the
   ITU-R BT.709 matrix (Kr = 0.2126, Kb = 0.0722; luma scale 255/219, chroma scale 255/224):
   cy = 1.16438 -> 1220945, V->R 1.79274 -> 1879825, V->G -0.53291 -> -558796,
   U->G -0.21325 -> -223607, U->B 2.11240 -> 2215014. */
void oracle_nv12_to_rgb(const uint8_t* yp, size_t y_pitch, const uint8_t* uvp, size_t uv_pitch,
                        uint32_t W, uint32_t H, int matrix, uint8_t* rgb) {
  const int32_t cy = matrix ? 1220945 : 1220542, vr = matrix ? 1879825 : 1673527;
  const int32_t vg = matrix ? -558796 : -852492, ug = matrix ? -223607 : -409993, ub = matrix ? 2215014 : 2116026;
  for (uint32_t y = 0; y < H; ++y) {
    for (uint32_t x = 0; x < W; ++x) {
      int32_t Y = yp[(size_t)y * y_pitch + x];
      int32_t U = uvp[(size_t)(y >> 1) * uv_pitch + 2 * (x >> 1)];
      int32_t V = uvp[(size_t)(y >> 1) * uv_pitch + 2 * (x >> 1) + 1];
      int32_t u = U - 128, v = V - 128;
      int32_t yy = (Y - 16 > 0 ? Y - 16 : 0) * cy;
      int32_t half = 1 << 19;
      uint8_t* px = rgb + ((size_t)y * W + x) * 3;
      px[0] = sat_u8((yy + half + vr * v) >> 20);
      px[1] = sat_u8((yy + half + vg * v + ug * u) >> 20);
      px[2] = sat_u8((yy + half + ub * u) >> 20);
    }
  }
}

/* ------------------------------------------------------------------------- */
/* O7. Bilinear resample (Fig. 9 P:L221-225 "bilinear"; R#12): half-pixel     */
/* centres, no antialias, clamp to the source, fp32 lerp, rint -> uint8 (Q2). */
/* ------------------------------------------------------------------------- */
static float lerp_tap(float lam, float a, float b) { return fmaf(lam, b - a, a); }

static uint8_t q_u8(float v) {
  float r = rintf(v);                      /* round half to even */
  if (r < 0.f) r = 0.f;
  if (r > 255.f) r = 255.f;
  return (uint8_t)r;
}

/* source coordinate of output index o for scale sc, as torch upsample_bilinear2d */
static float src_coord(float sc, float o) {
  float s = sc * (o + 0.5f) - 0.5f;        /* two separately rounded ops (no contraction) */
  return s > 0.f ? s : 0.f;
}

/* img: HWC u8 of size w x h (already the crop). out: Ho x Wo x 3. */
void oracle_resize(const uint8_t* img, uint32_t w, uint32_t h, uint32_t Ho, uint32_t Wo, uint8_t* out) {
  float scx = (float)w / (float)Wo;
  float scy = (float)h / (float)Ho;
  for (uint32_t oy = 0; oy < Ho; ++oy) {
    float sy = src_coord(scy, (float)oy);
    uint32_t y0 = (uint32_t)sy;
    float ly = sy - (float)y0;
    uint32_t y1 = y0 + 1 < h ? y0 + 1 : h - 1;
    for (uint32_t ox = 0; ox < Wo; ++ox) {
      float sx = src_coord(scx, (float)ox);
      uint32_t x0 = (uint32_t)sx;
      float lx = sx - (float)x0;
      uint32_t x1 = x0 + 1 < w ? x0 + 1 : w - 1;
      for (int c = 0; c < 3; ++c) {
        float p00 = img[((size_t)y0 * w + x0) * 3 + c];
        float p01 = img[((size_t)y0 * w + x1) * 3 + c];
        float p10 = img[((size_t)y1 * w + x0) * 3 + c];
        float p11 = img[((size_t)y1 * w + x1) * 3 + c];
        float h0 = lerp_tap(lx, p00, p01);
        float h1 = lerp_tap(lx, p10, p11);
        out[((size_t)oy * Wo + ox) * 3 + c] = q_u8(lerp_tap(ly, h0, h1));
      }
    }
  }
}

/* RRC = crop then resize (torchvision resized_crop). rgb: W x H HWC. */
void oracle_resized_crop(const uint8_t* rgb, uint32_t W, uint32_t H, const int32_t box[4],
                         uint32_t Ho, uint32_t Wo, uint8_t* out) {
  (void)H;
  uint32_t x0 = (uint32_t)box[0], y0 = (uint32_t)box[1], w = (uint32_t)box[2], h = (uint32_t)box[3];
  uint8_t* crop = (uint8_t*)malloc((size_t)w * h * 3);
  for (uint32_t y = 0; y < h; ++y)
    memcpy(crop + (size_t)y * w * 3, rgb + ((size_t)(y0 + y) * W + x0) * 3, (size_t)w * 3);
  oracle_resize(crop, w, h, Ho, Wo, out);
  free(crop);
}

/* SHORTSIDE_CROP = resize the whole frame to W' x H', then crop Ho x Wo at (x_off, y_off).
   Evaluated pointwise: identical to materialising the W' x H' image then cropping. */
void oracle_shortside_crop(const uint8_t* rgb, uint32_t W, uint32_t H, const int32_t box[4],
                           uint32_t Ho, uint32_t Wo, uint8_t* out) {
  uint32_t xo = (uint32_t)box[0], yo = (uint32_t)box[1], Wp = (uint32_t)box[2], Hp = (uint32_t)box[3];
  uint8_t* full = (uint8_t*)malloc((size_t)Wp * Hp * 3);
  oracle_resize(rgb, W, H, Hp, Wp, full);
  for (uint32_t y = 0; y < Ho; ++y)
    memcpy(out + (size_t)y * Wo * 3, full + ((size_t)(yo + y) * Wp + xo) * 3, (size_t)Wo * 3);
  free(full);
}

/* O8. Horizontal flip (Fig. 9): out[y][x] = in[y][Wo-1-x]. */
void oracle_flip(const uint8_t* in, uint32_t Ho, uint32_t Wo, uint8_t* out) {
  for (uint32_t y = 0; y < Ho; ++y)
    for (uint32_t x = 0; x < Wo; ++x)
      for (int c = 0; c < 3; ++c)
        out[((size_t)y * Wo + x) * 3 + c] = in[((size_t)y * Wo + (Wo - 1 - x)) * 3 + c];
}

/* ------------------------------------------------------------------------- */
/* O9. Rotation about the image centre (R#15): torchvision     */
/* F.rotate(img, theta, BILINEAR, fill=None) semantics, zero outside, rint.   */
/* ------------------------------------------------------------------------- */
void oracle_rotate(const uint8_t* in, uint32_t Ho, uint32_t Wo, double theta_deg, uint8_t* out) {
  const double pi = 3.14159265358979323846;
  float c = (float)cos(theta_deg * pi / 180.0);
  float s = (float)sin(theta_deg * pi / 180.0);
  float ns = -s;
  float cx = (float)(Wo - 1) * 0.5f;
  float cy = (float)(Ho - 1) * 0.5f;
  for (uint32_t oy = 0; oy < Ho; ++oy) {
    for (uint32_t ox = 0; ox < Wo; ++ox) {
      float xc = (float)ox - cx;
      float yc = (float)oy - cy;
      float sx = (c * xc + ns * yc) + cx;    /* inverse map: output pixel -> input position */
      float sy = (s * xc + c * yc) + cy;
      float fx0 = floorf(sx), fy0 = floorf(sy);
      float lx = sx - fx0, ly = sy - fy0;
      int32_t x0 = (int32_t)fx0, y0 = (int32_t)fy0;
      for (int ch = 0; ch < 3; ++ch) {
        float p[2][2];
        for (int dy = 0; dy < 2; ++dy)
          for (int dx = 0; dx < 2; ++dx) {
            int32_t xx = x0 + dx, yy = y0 + dy;
            int inside = xx >= 0 && xx < (int32_t)Wo && yy >= 0 && yy < (int32_t)Ho;
            p[dy][dx] = inside ? (float)in[((size_t)yy * Wo + (size_t)xx) * 3 + ch] : 0.f;
          }
        float h0 = lerp_tap(lx, p[0][0], p[0][1]);
        float h1 = lerp_tap(lx, p[1][0], p[1][1]);
        out[((size_t)oy * Wo + ox) * 3 + ch] = q_u8(lerp_tap(ly, h0, h1));
      }
    }
  }
}

/* ------------------------------------------------------------------------- */
/* O10. Separable Gaussian blur ("blurring"; R#16): radius r, weights   */
/* exp(-(i-r)^2 / (2 sigma^2)) normalised in double then cast to float,       */
/* horizontal then vertical, reflect border, fp32 accumulation, rint.         */
/* ------------------------------------------------------------------------- */
void oracle_blur_weights(double sigma, uint32_t r, float* w) {
  double tmp[64];
  double sum = 0.0;
  for (uint32_t i = 0; i <= 2 * r; ++i) {
    double d = (double)i - (double)r;
    tmp[i] = exp(-(d * d) / (2.0 * sigma * sigma));
    sum += tmp[i];
  }
  for (uint32_t i = 0; i <= 2 * r; ++i) w[i] = (float)(tmp[i] / sum);
}

static int32_t reflect(int32_t p, int32_t n) {   /* ... c b | a b c ... (torch "reflect") */
  if (p < 0) return -p;
  if (p >= n) return 2 * (n - 1) - p;
  return p;
}

void oracle_blur(const uint8_t* in, uint32_t Ho, uint32_t Wo, double sigma, uint32_t r, uint8_t* out) {
  float w[64];
  oracle_blur_weights(sigma, r, w);
  float* tmp = (float*)malloc(sizeof(float) * (size_t)Ho * Wo * 3);
  for (uint32_t y = 0; y < Ho; ++y)              /* horizontal pass -> fp32 */
    for (uint32_t x = 0; x < Wo; ++x)
      for (int c = 0; c < 3; ++c) {
        float acc = 0.f;
        for (uint32_t i = 0; i <= 2 * r; ++i) {
          int32_t xx = reflect((int32_t)x + (int32_t)i - (int32_t)r, (int32_t)Wo);
          acc = fmaf(w[i], (float)in[((size_t)y * Wo + (size_t)xx) * 3 + c], acc);
        }
        tmp[((size_t)y * Wo + x) * 3 + c] = acc;
      }
  for (uint32_t y = 0; y < Ho; ++y)              /* vertical pass -> rint -> u8 */
    for (uint32_t x = 0; x < Wo; ++x)
      for (int c = 0; c < 3; ++c) {
        float acc = 0.f;
        for (uint32_t i = 0; i <= 2 * r; ++i) {
          int32_t yy = reflect((int32_t)y + (int32_t)i - (int32_t)r, (int32_t)Ho);
          acc = fmaf(w[i], tmp[((size_t)yy * Wo + x) * 3 + c], acc);
        }
        out[((size_t)y * Wo + x) * 3 + c] = q_u8(acc);
      }
  free(tmp);
}

/* ------------------------------------------------------------------------- */
/* O11. Normalise + cast (north_star "mean/std normalisation into bf16/fp32") */
/* a_c = 1/(255 std_c), b_c = -mean_c/std_c in double, cast once; y = fma.    */
/* ------------------------------------------------------------------------- */
void oracle_norm_coeffs(const double mean[3], const double std[3], float a[3], float b[3]) {
  for (int c = 0; c < 3; ++c) {
    a[c] = (float)(1.0 / (255.0 * std[c]));
    b[c] = (float)(-mean[c] / std[c]);
  }
}

float oracle_normalize(uint8_t q, float a, float b) { return fmaf((float)q, a, b); }

uint16_t oracle_bf16_rne(float f) {               /* round to nearest even (finite inputs) */
  uint32_t u;
  memcpy(&u, &f, 4);
  uint32_t lsb = (u >> 16) & 1u;
  u += 0x7fffu + lsb;
  return (uint16_t)(u >> 16);
}

/* ------------------------------------------------------------------------- */
/* Colour jitter ("colour jitter"; R#30), on an HWC uint8 image in place, */
/* after flip and before rotation (op order R#14 + R#30). torchvision's         */
/* adjust_brightness / adjust_contrast / adjust_saturation on uint8 tensors,     */
/* written out with every float32 operation rounded on its own:                 */
/*   brightness f: o = trunc(clamp(x * f, 0, 255))                               */
/*   gray(r,g,b) = floor((r * 0.2989f + g * 0.587f) + b * 0.114f)                */
/*   saturation f: o = trunc(clamp(x * f + gray * (float)(1 - f), 0, 255))       */
/*   contrast f:   m = (float)sum(gray) / (float)(H W) (an exact integer sum),   */
/*                 o = trunc(clamp(x * f + m * (float)(1 - f), 0, 255))          */
/* order k = 0..5 is the k-th permutation of (brightness, contrast, saturation)  */
/* in lexicographic order.                                                       */
/* ------------------------------------------------------------------------- */
static float jit_gray(uint8_t r, uint8_t g, uint8_t b) {
  float t = (float)r * 0.2989f;
  t = t + (float)g * 0.587f;
  t = t + (float)b * 0.114f;
  return floorf(t);
}
static uint8_t jit_u8(float v) {
  if (v < 0.f) v = 0.f;
  if (v > 255.f) v = 255.f;
  return (uint8_t)v;            /* truncation toward zero, like torch's float -> uint8 */
}
void oracle_color_jitter(uint8_t* img, uint32_t H, uint32_t W, const double f[3], uint32_t order) {
  static const int perm[6][3] = {{0, 1, 2}, {0, 2, 1}, {1, 0, 2}, {1, 2, 0}, {2, 0, 1}, {2, 1, 0}};
  size_t n = (size_t)H * W;
  for (int s = 0; s < 3; ++s) {
    int op = perm[order % 6][s];
    float fx = (float)f[op], fa = (float)(1.0 - f[op]);
    if (op == 0) {
      for (size_t i = 0; i < 3 * n; ++i) img[i] = jit_u8((float)img[i] * fx);
    } else if (op == 1) {
      uint64_t sum = 0;
      for (size_t i = 0; i < n; ++i) sum += (uint64_t)jit_gray(img[3 * i], img[3 * i + 1], img[3 * i + 2]);
      float mean = (float)sum / (float)n;
      for (size_t i = 0; i < 3 * n; ++i) img[i] = jit_u8((float)img[i] * fx + mean * fa);
    } else {
      for (size_t i = 0; i < n; ++i) {
        float gr = jit_gray(img[3 * i], img[3 * i + 1], img[3 * i + 2]);
        for (int c = 0; c < 3; ++c) img[3 * i + c] = jit_u8((float)img[3 * i + c] * fx + gr * fa);
      }
    }
  }
}

/* ------------------------------------------------------------------------- */
/* Render one output frame (view k, time t) of one planned clip:              */
/* NV12 -> RGB (Q1) -> crop/resize (Q2) -> flip -> rotate (Q3) -> blur (Q4)   */
/* -> normalise -> out[c][y][x] in the view's dtype (op order R#14).          */
/* ------------------------------------------------------------------------- */
void oracle_render_frame(const oracle_spec* spec, const oracle_clip_meta* meta, uint32_t k,
                         const uint8_t* yp, size_t y_pitch, const uint8_t* uvp, size_t uv_pitch,
                         uint32_t W, uint32_t H, void* out_chw) {
  const oracle_view* v = &spec->views[k];
  uint32_t q = v->spatial_group;
  uint32_t Ho = v->out_h, Wo = v->out_w;
  size_t n = (size_t)Ho * Wo * 3;
  uint8_t* rgb = (uint8_t*)malloc((size_t)W * H * 3);
  uint8_t* a = (uint8_t*)malloc(n);
  uint8_t* b = (uint8_t*)malloc(n);
  oracle_nv12_to_rgb(yp, y_pitch, uvp, uv_pitch, W, H, v->color_matrix, rgb);
  if (v->geom == OR_GEOM_RRC)
    oracle_resized_crop(rgb, W, H, meta->box[q], Ho, Wo, a);
  else
    oracle_shortside_crop(rgb, W, H, meta->box[q], Ho, Wo, a);
  if (meta->flip[q]) { oracle_flip(a, Ho, Wo, b); memcpy(a, b, n); }
  if (meta->jitter_on[q]) oracle_color_jitter(a, Ho, Wo, meta->jitter_f[q], meta->jitter_order[q]);
  if (meta->rot_on[q]) { oracle_rotate(a, Ho, Wo, meta->theta[q], b); memcpy(a, b, n); }
  if (meta->blur_on[q]) { oracle_blur(a, Ho, Wo, meta->sigma[q], meta->blur_r[q], b); memcpy(a, b, n); }
  float ca[3], cb[3];
  oracle_norm_coeffs(v->mean, v->std, ca, cb);
  for (uint32_t c = 0; c < 3; ++c)
    for (uint32_t y = 0; y < Ho; ++y)
      for (uint32_t x = 0; x < Wo; ++x) {
        uint8_t qv = a[((size_t)y * Wo + x) * 3 + c];
        size_t o = ((size_t)c * Ho + y) * Wo + x;
        if (v->out_dtype == OR_U8) {
          ((uint8_t*)out_chw)[o] = qv;
        } else if (v->out_dtype == OR_BF16) {
          ((uint16_t*)out_chw)[o] = oracle_bf16_rne(oracle_normalize(qv, ca[c], cb[c]));
        } else {
          ((float*)out_chw)[o] = oracle_normalize(qv, ca[c], cb[c]);
        }
      }
  free(rgb);
  free(a);
  free(b);
}

/* ------------------------------------------------------------------------- */
/* Whole batch: out[k] is view k's [B][3][T_k][Ho][Wo] tensor (O12 layout).   */
/* frames[] holds every (video, frame) the batch needs (any order).           */
/* ------------------------------------------------------------------------- */
typedef struct {
  uint32_t video, frame, width, height;
  const uint8_t* y;
  const uint8_t* uv;
  uint64_t y_pitch, uv_pitch;
} oracle_frame_ref;

static size_t dtype_size(int32_t d) { return d == OR_U8 ? 1 : (d == OR_BF16 ? 2 : 4); }

int oracle_materialize(const oracle_spec* spec, const oracle_video_info* dataset, uint32_t n_videos,
                       uint64_t epoch, uint32_t rank, uint64_t iteration, const oracle_frame_ref* frames,
                       uint32_t n_frame_refs, void* const* out, oracle_clip_meta* metas) {
  int rc = oracle_plan_batch(spec, dataset, n_videos, epoch, rank, iteration, metas);
  if (rc) return rc;
  for (uint32_t b = 0; b < spec->batch_size; ++b) {
    for (uint32_t k = 0; k < spec->n_views; ++k) {
      const oracle_view* v = &spec->views[k];
      size_t es = dtype_size(v->out_dtype);
      size_t plane = (size_t)v->out_h * v->out_w;
      uint8_t* chw = (uint8_t*)malloc(plane * 3 * es);
      for (uint32_t t = 0; t < v->clip_len; ++t) {
        const oracle_frame_ref* fr = NULL;
        for (uint32_t i = 0; i < n_frame_refs; ++i)
          if (frames[i].video == metas[b].video && frames[i].frame == metas[b].frames[k][t]) fr = &frames[i];
        if (fr == NULL) { free(chw); return -2; }
        oracle_render_frame(spec, &metas[b], k, fr->y, fr->y_pitch, fr->uv, fr->uv_pitch, fr->width,
                            fr->height, chw);
        for (uint32_t c = 0; c < 3; ++c) {
          size_t dst = ((((size_t)b * 3 + c) * v->clip_len + t) * plane) * es;
          memcpy((uint8_t*)out[k] + dst, chw + (size_t)c * plane * es, plane * es);
        }
      }
      free(chw);
    }
  }
  return 0;
}

/* ------------------------------------------------------------------------- */
/* O13. Algorithmic source bytes of one batch: the number of distinct 32-byte */
/* sectors of (video, frame, plane, row) touched by the bilinear taps of any  */
/* view, deduplicated across views and groups (rows assumed 32 B aligned).    */
/* O14. Reuse accounting: fetches = batch-unique source frames,  */
/* uses = output frames (view, clip, t).                                      */
/* ------------------------------------------------------------------------- */
typedef struct {
  uint64_t src_sectors;      /* O13 */
  uint64_t out_bytes;
  uint64_t fetches;          /* O14 */
  uint64_t uses;
} oracle_batch_bytes;

static void mark_taps_1d(float sc, uint32_t n_out, uint32_t offset, uint32_t clamp_n, int flip_unused,
                         uint8_t* used) {
  (void)flip_unused;
  for (uint32_t o = 0; o < n_out; ++o) {
    float s = src_coord(sc, (float)(offset + o));
    uint32_t i0 = (uint32_t)s;
    uint32_t i1 = i0 + 1 < clamp_n ? i0 + 1 : clamp_n - 1;
    used[i0] = 1;
    used[i1] = 1;
  }
}

int oracle_batch_bytes_of(const oracle_spec* spec, const oracle_video_info* dataset, uint32_t n_videos,
                          uint64_t epoch, uint32_t rank, uint64_t iteration, oracle_batch_bytes* res) {
  uint32_t B = spec->batch_size;
  oracle_clip_meta* metas = (oracle_clip_meta*)malloc(sizeof(oracle_clip_meta) * B);
  int rc = oracle_plan_batch(spec, dataset, n_videos, epoch, rank, iteration, metas);
  if (rc) { free(metas); return rc; }
  memset(res, 0, sizeof(*res));
  /* list of distinct (video, frame) used by the batch */
  uint32_t cap = B * OR_MAX_VIEWS * OR_MAX_T;
  uint32_t* fv = (uint32_t*)malloc(sizeof(uint32_t) * cap);
  uint32_t* ff = (uint32_t*)malloc(sizeof(uint32_t) * cap);
  uint32_t nf = 0;
  for (uint32_t b = 0; b < B; ++b)
    for (uint32_t k = 0; k < spec->n_views; ++k) {
      const oracle_view* v = &spec->views[k];
      res->uses += v->clip_len;
      res->out_bytes += (uint64_t)v->clip_len * 3 * v->out_h * v->out_w * dtype_size(v->out_dtype);
      for (uint32_t t = 0; t < v->clip_len; ++t) {
        uint32_t vid = metas[b].video, fr = metas[b].frames[k][t], seen = 0;
        for (uint32_t i = 0; i < nf; ++i)
          if (fv[i] == vid && ff[i] == fr) seen = 1;
        if (!seen) { fv[nf] = vid; ff[nf] = fr; ++nf; }
      }
    }
  res->fetches = nf;
  for (uint32_t i = 0; i < nf; ++i) {
    const oracle_video_info* vi = NULL;
    for (uint32_t d = 0; d < n_videos; ++d)
      if (dataset[d].video == fv[i]) vi = &dataset[d];
    uint32_t W = vi->width, H = vi->height;
    uint8_t* touched = (uint8_t*)calloc((size_t)W * H, 1);      /* luma pixels touched by a tap */
    for (uint32_t b = 0; b < B; ++b) {
      if (metas[b].video != fv[i]) continue;
      for (uint32_t k = 0; k < spec->n_views; ++k) {
        const oracle_view* v = &spec->views[k];
        int uses_frame = 0;
        for (uint32_t t = 0; t < v->clip_len; ++t)
          if (metas[b].frames[k][t] == ff[i]) uses_frame = 1;
        if (!uses_frame) continue;
        const int32_t* box = metas[b].box[v->spatial_group];
        uint8_t* cols = (uint8_t*)calloc(W, 1);
        uint8_t* rows = (uint8_t*)calloc(H, 1);
        if (v->geom == OR_GEOM_RRC) {
          uint8_t* c2 = (uint8_t*)calloc((size_t)box[2], 1);
          uint8_t* r2 = (uint8_t*)calloc((size_t)box[3], 1);
          mark_taps_1d((float)box[2] / (float)v->out_w, v->out_w, 0, (uint32_t)box[2], 0, c2);
          mark_taps_1d((float)box[3] / (float)v->out_h, v->out_h, 0, (uint32_t)box[3], 0, r2);
          for (int32_t x = 0; x < box[2]; ++x) if (c2[x]) cols[box[0] + x] = 1;
          for (int32_t y = 0; y < box[3]; ++y) if (r2[y]) rows[box[1] + y] = 1;
          free(c2);
          free(r2);
        } else {
          mark_taps_1d((float)W / (float)box[2], v->out_w, (uint32_t)box[0], W, 0, cols);
          mark_taps_1d((float)H / (float)box[3], v->out_h, (uint32_t)box[1], H, 0, rows);
        }
        for (uint32_t y = 0; y < H; ++y)
          if (rows[y])
            for (uint32_t x = 0; x < W; ++x)
              if (cols[x]) touched[(size_t)y * W + x] = 1;
        free(cols);
        free(rows);
      }
    }
    /* Y plane sectors: (row, x/32); UV plane sectors: (row/2, (2*(x/2))/32) for U and V bytes */
    uint32_t nsec = (W + 31) / 32;
    uint8_t* ysec = (uint8_t*)calloc((size_t)H * nsec, 1);
    uint8_t* uvsec = (uint8_t*)calloc((size_t)(H / 2) * nsec, 1);
    for (uint32_t y = 0; y < H; ++y)
      for (uint32_t x = 0; x < W; ++x)
        if (touched[(size_t)y * W + x]) {
          ysec[(size_t)y * nsec + x / 32] = 1;
          uvsec[(size_t)(y / 2) * nsec + (2 * (x / 2)) / 32] = 1;     /* U byte */
          uvsec[(size_t)(y / 2) * nsec + (2 * (x / 2) + 1) / 32] = 1; /* V byte */
        }
    for (size_t s = 0; s < (size_t)H * nsec; ++s) res->src_sectors += ysec[s];
    for (size_t s = 0; s < (size_t)(H / 2) * nsec; ++s) res->src_sectors += uvsec[s];
    free(ysec);
    free(uvsec);
    free(touched);
  }
  free(fv);
  free(ff);
  free(metas);
  return 0;
}

/* struct sizes for the Python wrapper's layout check */
size_t oracle_sizeof_spec(void) { return sizeof(oracle_spec); }
size_t oracle_sizeof_meta(void) { return sizeof(oracle_clip_meta); }
size_t oracle_sizeof_frame_ref(void) { return sizeof(oracle_frame_ref); }
