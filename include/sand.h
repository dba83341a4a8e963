/*
 * sand.h — C-ABI of the B200-native SAND view-materialisation library (libsand.so).
 *
 * SAND (SOSP'25, /root/reference/PAPER.md) exposes training batches as *views*:
 * virtual objects materialised when accessed (§5.1), addressed as
 * /{task}/{epoch}/{iteration}/view (Table 1) and used through
 * open / read / getxattr / close (Table 2). This library is that view
 * abstraction for the per-batch materialisation hot path (BASELINE.json
 * north_star), with decoded frames resident in an HBM frame store:
 *
 *   paper                                  this ABI
 *   decoded frame objects (Table 1)  sand_store_* (HBM, keyed by (video, frame))
 *   open(view path)        sand_view_create
 *   read(fd)        sand_view_read_batch(view, epoch, rank, out)
 *   getxattr(path, meta)  sand_view_get_meta
 *   close(fd)        sand_view_destroy
 *
 * Conventions
 *  - Every function returns int: SAND_OK (0) or a negative SAND_E* code; nothing
 *    throws across the ABI. sand_last_error() gives a thread-local message.
 *  - Pointers named "device" are CUDA device addresses on the store's device;
 *    everything else is host memory. Streams are cudaStream_t passed as void*
 *    (NULL = the legacy default stream). Asynchronous calls are ordered on the
 *    given stream; the caller keeps sources alive until the stream reaches them.
 *  - One handle must not be used from two threads at once; distinct handles are
 *    independent.
 *  - Output of sand_view_read_batch is a pure function of (store bytes, spec,
 *    epoch, rank, iteration); per clip it does not depend on world_size or rank
 *    (RNG counters use global clip ids; R#1).
 */
#ifndef SAND_H
#define SAND_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define SAND_MAX_VIEWS 8   /* views (tasks / trials / pathways) per view group */
#define SAND_MAX_GROUPS 8  /* spatial groups; group ids are 0..7 */
#define SAND_MAX_T 64      /* frames per clip per view */

enum {
  SAND_OK = 0,
  SAND_EINVAL = -1, /* invalid argument / spec (odd NV12 dims, alignment, crop > frame, ...) */
  SAND_ENOENT = -2, /* a planned (video, frame) is not in the store */
  SAND_ENOMEM = -3, /* store capacity or allocation failure */
  SAND_ERANGE = -4, /* iteration >= sand_view_iterations, or video id unknown */
  SAND_ECUDA = -5,  /* CUDA runtime error (message in sand_last_error) */
  SAND_EBUSY = -6   /* store still has live views */
};
enum { SAND_U8 = 0, SAND_BF16 = 1, SAND_F32 = 2 };             /* output dtypes */
enum { SAND_GEOM_RRC = 0, SAND_GEOM_SHORTSIDE_CROP = 1 };      /* view geometry */
enum { SAND_BT601 = 0, SAND_BT709 = 1 };                        /* YUV -> RGB matrix (R#11, R#29) */

typedef struct sand_store sand_store; /* opaque; owns the device frame slab */
typedef struct sand_view sand_view;   /* opaque; a view group over one clip stream */
typedef void* sand_stream_t;          /* cudaStream_t */

/* ------------------------------------------------------------------ store */

/* Create a frame store on `cuda_device` owning one device slab of capacity_bytes.
 * *out receives the handle. Errors: EINVAL, ENOMEM, ECUDA. */
int sand_store_create(int cuda_device, uint64_t capacity_bytes, sand_store** out);

/* Reserve slab space for video `video` with n_frames NV12 frames of width x height
 * (both even). Each frame is laid out as H rows of the Y plane then H/2 rows of
 * interleaved UV, row pitch = width rounded up to 64 B, frame stride a multiple of
 * 256 B. Errors: EINVAL (odd/zero dims, video already added with other dims),
 * ENOMEM (capacity). Re-adding with identical dims is a no-op. */
int sand_store_add_video(sand_store* s, uint32_t video, uint32_t n_frames, uint32_t width,
                         uint32_t height);

/* Copy frames [first_frame, first_frame + n_frames) of a video into the store,
 * stream-ordered. y/uv point at the first frame's Y and UV planes; consecutive
 * frames are y_frame_stride / uv_frame_stride bytes apart; rows are y_pitch /
 * uv_pitch apart. src_on_device != 0: y/uv are device pointers, else host (pinned
 * host memory makes the copy asynchronous). Putting a frame again overwrites it
 * and resets its counters. Ordering: every put records a store event on `stream`
 * (after waiting on the previous put's event, so puts on different streams are
 * chained), and a later sand_view_read_batch on ANY stream waits on it before its
 * kernels, so a read never consumes a frame whose copy has not landed. Errors: ERANGE
 * (unknown video / frame range), EINVAL, ECUDA. */
int sand_store_put_frames(sand_store* s, uint32_t video, uint32_t first_frame, uint32_t n_frames,
                          const uint8_t* y, uint64_t y_pitch, uint64_t y_frame_stride,
                          const uint8_t* uv, uint64_t uv_pitch, uint64_t uv_frame_stride,
                          int src_on_device, sand_stream_t stream);

/* Copy n frames of possibly different videos into the store in one call: frame i is
 * (videos[i], frames[i]); its Y plane starts at src + i * frame_stride (rows `pitch` bytes
 * apart) and its interleaved UV plane at src + i * frame_stride + uv_offset (same pitch).
 * All n frames must have the same width/height (their videos' dims). This is the
 * decoder-output path of the store (§6: decoded frames become objects of the
 * store): a host source (src_on_device == 0; pinned memory keeps it asynchronous) is
 * moved with ONE host->device copy into a store-owned staging buffer, then one scatter
 * kernel writes every frame into its pitched slot; a device source is scattered directly.
 * Stream-ordered on `stream`; the caller keeps src valid until the stream reaches the
 * copy. The call waits (host side) until the previous batch put's scatter has run, so
 * the staging buffer is never overwritten while still being read. Putting a frame again
 * overwrites it and resets its counters. Ordered before later reads exactly as
 * sand_store_put_frames. Nothing is copied if any (video, frame) is unknown. Errors: ERANGE (unknown video / frame), EINVAL (null pointers, frames of
 * different sizes, pitch/uv_offset/frame_stride too small), ECUDA. */
int sand_store_put_frame_batch(sand_store* s, uint32_t n, const uint32_t* videos, const uint32_t* frames,
                               const uint8_t* src, uint64_t frame_stride, uint64_t pitch, uint64_t uv_offset,
                               int src_on_device, sand_stream_t stream);

/* Device address and layout of one stored frame (for tests / zero-copy producers such
 * as a decoder writing NV12 in place). Errors: ERANGE. */
typedef struct {
  uint64_t y;          /* device address of the Y plane */
  uint64_t uv;         /* device address of the UV plane */
  uint32_t pitch;      /* row pitch of both planes, bytes */
  uint32_t width, height, n_frames;
  uint64_t frame_stride;
} sand_frame_layout;
int sand_store_frame_layout(const sand_store* s, uint32_t video, uint32_t frame,
                            sand_frame_layout* out);

/* Mark frames as present without copying (after a producer wrote them in place via
 * sand_store_frame_layout). The store cannot see those writes: the caller orders them
 * before later sand_view_read_batch calls (same stream, or an event the read stream
 * waits on). Errors: ERANGE. */
int sand_store_mark_present(sand_store* s, uint32_t video, uint32_t first_frame, uint32_t n_frames);

/* Reuse accounting (Fig. 16 / Fig. 19): totals over the store. A
 * "fetch" is one batch-unique source frame read by a read_batch; a "use" is one
 * output frame (view, clip, t) produced from it. */
typedef struct {
  uint64_t videos, frames_present, bytes_reserved, capacity;
  uint64_t fetches, uses, batches;
} sand_counters;
int sand_store_counters(const sand_store* s, sand_counters* out);

/* Per-frame counters of one video, frames [first, first + n). Errors: ERANGE. */
int sand_store_frame_counters(const sand_store* s, uint32_t video, uint32_t first, uint32_t n,
                              uint64_t* fetches, uint64_t* uses);

/* Free the store. EBUSY while views created on it are alive. */
int sand_store_destroy(sand_store* s);

/* ------------------------------------------------------------------ views */

/* One view: a task, a Ray trial or a SlowFast pathway (P:L180-182 config fields). */
typedef struct {
  uint32_t clip_len;        /* T frames per clip (<= SAND_MAX_T)                        */
  uint32_t stride;          /* temporal stride (P:L180 frame_stride)                    */
  int32_t pool_offset;      /* -1: random grid offset in the shared pool; >= 0 fixed (R#5) */
  uint32_t spatial_group;   /* 0..7: views with equal group share spatial draws (R#6);
                               they must agree on every spatial/augmentation field below */
  int32_t geom;             /* SAND_GEOM_RRC or SAND_GEOM_SHORTSIDE_CROP                */
  double scale_min, scale_max, ratio_min, ratio_max;   /* RRC ranges (R#8)               */
  uint32_t short_side;      /* SHORTSIDE_CROP: short side S before the crop (R#10)      */
  uint32_t out_h, out_w;    /* output frame size                                        */
  double flip_p;            /* horizontal flip probability (Fig. 9)          */
  double rot_p, rot_max_deg;            /* rotation gate and range (R#15)               */
  double blur_p, sigma_min, sigma_max;  /* blur gate and sigma range (R#16)             */
  uint32_t blur_ksize;      /* odd; radius cap (k-1)/2                                  */
  double blur_truncate;     /* radius = min((k-1)/2, floor(truncate*sigma+0.5)); 0 = cap  */
  double mean[3], std[3];   /* per-channel normalisation (R#17)                         */
  int32_t out_dtype;        /* SAND_U8 / SAND_BF16 / SAND_F32                           */
  int32_t subsample_of;     /* -1: frames from the shared pool (R#4, R#5). k >= 0: this view's
                               T frames are view k's frames at positions floor(t (T_k - 1) / (T - 1))
                               (PySlowFast linspace slow pathway); view k
                               must itself draw from the pool; stride/pool_offset are unused */
  int32_t color_matrix;     /* SAND_BT601 (R#11, OpenCV's integer form) or SAND_BT709 (R#29); every
                               view of a spec uses the same matrix (the decoder's colour space) */
  double jitter_p;          /* colour jitter gate (R#30): brightness, contrast and saturation */
  double brightness, contrast, saturation;   /* magnitudes m: factor ~ U[max(0, 1 - m), 1 + m]  */
} sand_view_desc;

typedef struct {
  uint64_t seed;
  uint32_t world_size, batch_size, samples_per_video;  /* B clips per rank per iteration */
  int32_t drop_last;        /* DistributedSampler drop_last (R#3)                      */
  const uint32_t* videos;   /* dataset: store video ids, in dataset order (host)        */
  uint32_t n_videos;
  uint32_t n_views;         /* 1..SAND_MAX_VIEWS                                        */
  int32_t shared_window;    /* P:L295 shared window across RRC groups (R#18)           */
  uint32_t pool_epochs;     /* k: a clip's shared frame pool is drawn once per chunk of
                               k epochs and reused by all of them ("decoded once and
                               cached for exactly k epochs"; R#25); 0 or 1: every epoch   */
  sand_view_desc views[SAND_MAX_VIEWS];
} sand_view_spec;

/* Create a view group on a store (the spec is copied). Validates the spec against
 * the store's videos. Errors: EINVAL, ERANGE (unknown video), ENOMEM, ECUDA. */
int sand_view_create(sand_store* s, const sand_view_spec* spec, sand_view** out);

/* Output tensor of view k: contiguous [B][3][T][out_h][out_w] of dtype. */
typedef struct {
  uint32_t dims[5];
  int32_t dtype;
  uint64_t bytes;
} sand_tensor_desc;
int sand_view_output_desc(const sand_view* v, uint32_t k, sand_tensor_desc* out);

/* Iterations per epoch for a rank (DistributedSampler num_samples / B, R#3). */
int sand_view_iterations(const sand_view* v, uint64_t epoch, uint32_t rank, uint64_t* n);

typedef struct {
  uint64_t iteration;                 /* the {iteration} of the view path (Table 1)   */
  sand_stream_t stream;               /* all device work is ordered on this stream    */
  void* data[SAND_MAX_VIEWS];         /* device outputs, 16 B aligned, see output_desc */
} sand_batch_out;

/* read(): materialise batch (epoch, rank, out->iteration) of every view into
 * out->data[k], asynchronously on out->stream. The epoch's plan is built on the host
 * on first use (or ahead of time by sand_view_prefetch_epoch) and uploaded once.
 * Errors (synchronous): EINVAL (null/misaligned outputs, rank >= world_size),
 * ERANGE (iteration), ENOENT (a planned frame is absent), ECUDA (launch failure). */
int sand_view_read_batch(sand_view* v, uint64_t epoch, uint32_t rank, const sand_batch_out* out);

/* Pre-materialisation (§5.4). sand_view_prematerialize runs the
 * kernels of batch (epoch, rank, iteration) AHEAD of its read, into a library-owned device
 * buffer, on the view's own low-priority stream, so they overlap whatever the caller's
 * streams are doing (the training step); it returns immediately. A later read of that batch
 * is served from the buffer: sand_view_read_batch makes out->stream wait for the batch and
 * copies it into out->data (device to device); or sand_view_acquire_batch hands the buffer
 * itself to the caller (data_out[k] = device pointer of view k, valid until
 * sand_view_release_batch; no copy). Results are bit-identical to a direct read.
 * sand_view_set_prematerialize(v, slots) allocates `slots` batch buffers (0 frees them; the
 * call waits for outstanding work). Errors: EINVAL (no slots configured, null pointers),
 * EBUSY (every slot holds a batch not yet read / released), ERANGE (acquire/release of a batch
 * that is not pre-materialised), plus read_batch's. */
int sand_view_set_prematerialize(sand_view* v, uint32_t slots);
int sand_view_prematerialize(sand_view* v, uint64_t epoch, uint32_t rank, uint64_t iteration);
int sand_view_acquire_batch(sand_view* v, uint64_t epoch, uint32_t rank, uint64_t iteration, sand_stream_t stream,
                            void* data_out[SAND_MAX_VIEWS]);
int sand_view_release_batch(sand_view* v, uint64_t epoch, uint32_t rank, uint64_t iteration, sand_stream_t stream);

/* HBM-budgeted object reuse (§5.3 Alg. 1, §6; DESIGN.md
 * R#27). The cached object is the RESIZED FRAME of a short-side view (R#10): the whole frame
 * resized to W' x H' (uint8 R, G, B planes), keyed by (video, frame). Any crop of it is a copy
 * plus normalisation, bit-identical to resampling the crop from the NV12 frame. read_batch
 * decides per item of a group whose leader view is SHORTSIDE_CROP without rotation/blur, in
 * batch order: HIT (cached: copied from the object), FILL (not cached, used again in a later
 * epoch of the k-epoch chunk — Alg. 1: caching the parent instead of its >= 2 leaves saves
 * space — and a slot is free after eviction: the resized frame is materialised into the cache,
 * then copied from), MISS (otherwise: resampled from the NV12 frame as usual). Eviction (§6),
 * down to 75 % of the budget when a fill finds no free slot (keeping the objects of the batch
 * being decided) and after each batch: first objects not needed again in the current chunk
 * (least recently used first), then the latest next use. One object size per view
 * (the first eligible item's W' x H'; others MISS). `bytes` = 0 disables the cache (default);
 * set it before the view plans or reads (EBUSY otherwise). Reads of a view with a cache must be
 * ordered among themselves (one stream, or the caller orders them). Errors: EINVAL (8 views,
 * mixed dtypes), EBUSY, ECUDA. */
int sand_view_set_object_budget(sand_view* v, uint64_t bytes);
typedef struct {
  uint64_t hits, fills, misses, evictions;   /* eligible items served by each path; objects evicted */
  uint64_t objects, bytes_used, bytes_budget;
  uint64_t decide_ns, stage_ns, launch_ns;   /* host time in read_batch: decisions, staging, launches */
} sand_object_stats;
int sand_view_object_stats(const sand_view* v, sand_object_stats* out);

/* Plan an epoch ahead of time on a background host thread (the plan analogue of
 * the paper's pre-materialisation threads). Returns immediately. */
int sand_view_prefetch_epoch(sand_view* v, uint64_t epoch, uint32_t rank);

/* getxattr(): per-clip metadata of a batch (frame indices, crop boxes, flip,
 * rotation, blur), written to out[0..B). Fields per group are indexed by group id. */
typedef struct {
  uint32_t clip;          /* global clip id (video index * S + sample) */
  uint32_t video, sample, pool_start;
  uint32_t frames[SAND_MAX_VIEWS][SAND_MAX_T];
  int32_t box[SAND_MAX_GROUPS][4];   /* RRC: x0,y0,w,h ; SHORTSIDE: x_off,y_off,W',H' */
  uint32_t flip[SAND_MAX_GROUPS], rot_on[SAND_MAX_GROUPS], blur_on[SAND_MAX_GROUPS],
      blur_r[SAND_MAX_GROUPS];
  double theta[SAND_MAX_GROUPS], sigma[SAND_MAX_GROUPS];
  uint32_t jitter_on[SAND_MAX_GROUPS], jitter_order[SAND_MAX_GROUPS];   /* R#30: order 0..5 of (B, C, S) */
  double jitter_f[SAND_MAX_GROUPS][3];                                  /* brightness, contrast, saturation */
} sand_clip_meta;
int sand_view_get_meta(sand_view* v, uint64_t epoch, uint32_t rank, uint64_t iteration,
                       sand_clip_meta* out);

/* Algorithmic bytes of one batch: distinct 32 B sectors of source
 * rows touched by bilinear taps (deduplicated across views and groups) and output
 * bytes; plus the reuse counts the batch adds. */
typedef struct {
  uint64_t src_sectors, src_bytes, out_bytes, fetches, uses;
} sand_batch_bytes;
int sand_view_batch_bytes(sand_view* v, uint64_t epoch, uint32_t rank, uint64_t iteration,
                          sand_batch_bytes* out);

/* Item classes of a batch (each launched as its own kernel): 0 = plain items with a source
 * step <= 2 on both axes (k_plain / k_copy / k_stream), 1 = plain items with heavier
 * down-scaling (k_direct), 2 = items with rotation and/or blur (k_stencil2). */
#define SAND_N_CLASSES 3

/* sand_view_batch_bytes restricted to the items of class `cls`: the sectors the class's own
 * taps touch (deduplicated within the class), the bytes its items write, its fetches and uses.
 * The per-kernel roofline numerator of the measurement. Errors: EINVAL, ERANGE. */
int sand_view_batch_bytes_class(sand_view* v, uint64_t epoch, uint32_t rank, uint64_t iteration, uint32_t cls,
                                sand_batch_bytes* out);

/* Per-class kernel timing (measurement only): with sand_view_set_timing(v, 1) every
 * read_batch records CUDA events around each class's kernel on the stream it is launched on;
 * sand_view_class_times waits for the recorded events and returns, per class, the summed
 * milliseconds and launch count since the previous call (then resets them). Timing is off by
 * default (read_batch records nothing). Errors: EINVAL, ECUDA. */
int sand_view_set_timing(sand_view* v, int on);
int sand_view_class_times(sand_view* v, double ms[SAND_N_CLASSES], uint64_t launches[SAND_N_CLASSES]);

/* Host-only planning (no store, no device): the same planner read_batch uses.
 * sand_plan_rank_clips writes the global clip ids of (epoch, rank) in DistributedSampler
 * order (R#2, R#3) to out[0..*n) (cap entries available); sand_plan_clip plans one clip
 * (temporal indices, spatial draws; R#4-R#18) given per-dataset-video frame counts and frame
 * sizes (arrays of spec->n_videos entries). Errors: EINVAL (spec), ERANGE (cap / clip). */
int sand_plan_rank_clips(const sand_view_spec* spec, uint64_t epoch, uint32_t rank, uint32_t* out, uint32_t cap,
                         uint32_t* n);
int sand_plan_clip(const sand_view_spec* spec, const uint32_t* n_frames, const uint32_t* widths,
                   const uint32_t* heights, uint64_t epoch, uint32_t clip, sand_clip_meta* out);

/* Statistics of a view group: batches read, kernels launched, epoch plans built and work
 * items launched so far; host time spent building plans (all builder threads), blocked in
 * read_batch waiting for a plan, and inside read_batch in total (nanoseconds); the planner's
 * CPU time alone, its waits for recycled plan buffers, read_batch's wait for the view lock,
 * and how many reads found their epoch plan still being built. */
typedef struct {
  uint64_t batches, kernel_launches, plans_built, work_items;
  uint64_t plan_build_ns, plan_wait_ns, read_ns;
  uint64_t plan_cpu_ns, plan_buffer_wait_ns, lock_wait_ns, pending_waits;
} sand_view_stats;
int sand_view_get_stats(const sand_view* v, sand_view_stats* out);

/* close(): free the view group (waits for its in-flight work). */
int sand_view_destroy(sand_view* v);

/* Thread-local description of the last error on this thread ("" if none). */
const char* sand_last_error(void);

/* Library version string. */
const char* sand_version(void);

/* sizeof of the public structs, for binding layout checks: sizes[0..7] =
 * sand_frame_layout, sand_counters, sand_view_desc, sand_view_spec, sand_tensor_desc,
 * sand_batch_out, sand_clip_meta, sand_batch_bytes. Returns the count written (8). */
int sand_abi_sizes(uint64_t sizes[8]);

#ifdef __cplusplus
}
#endif
#endif /* SAND_H */
