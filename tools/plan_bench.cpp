// plan_bench.cpp — host-only timing of the epoch planner (build_plan) on a synthetic store
// description (no device memory is touched). Build + run:
//   python tools/plan_bench.py            (compiles against the in-tree libsand.so)
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>

#include "internal.h"

int main(int argc, char** argv) {
  const char* cfg = argc > 1 ? argv[1] : "k400";
  const int reps = argc > 2 ? std::atoi(argv[2]) : 20;
  sand_store store;
  sand_view v;
  v.store = &store;
  sand_view_spec& s = v.info.spec;
  std::memset(&s, 0, sizeof(s));
  s.seed = 0;
  s.world_size = 1;
  s.samples_per_video = 1;
  const bool sf = std::strcmp(cfg, "slowfast") == 0;
  s.batch_size = sf ? 16 : 32;
  s.n_views = sf ? 2 : 1;
  for (uint32_t k = 0; k < s.n_views; ++k) {
    sand_view_desc& d = s.views[k];
    d.clip_len = sf ? (k == 0 ? 32 : 8) : 16;
    d.stride = sf ? (k == 0 ? 2 : 8) : 4;
    d.pool_offset = sf ? 0 : -1;
    d.geom = sf ? SAND_GEOM_SHORTSIDE_CROP : SAND_GEOM_RRC;
    d.short_side = sf ? 256 : 0;
    d.scale_min = 0.08, d.scale_max = 1.0, d.ratio_min = 0.75, d.ratio_max = 4.0 / 3.0;
    d.out_h = d.out_w = 224;
    d.flip_p = 0.5;
    d.sigma_min = 0.1, d.sigma_max = 2.0, d.blur_ksize = 23, d.blur_truncate = 4.0;
    for (int c = 0; c < 3; ++c) d.mean[c] = 0.45, d.std[c] = 0.225;
    d.out_dtype = SAND_BF16;
  }
  const uint32_t n_videos = 1024;
  for (uint32_t i = 0; i < n_videos; ++i) {
    sand::VideoEntry& e = store.videos[i];
    e.id = i, e.n_frames = 300, e.width = 340, e.height = 256, e.pitch = 384;
    e.frame_stride = 384 * 384, e.offset = (uint64_t)i * 300 * e.frame_stride;
    v.info.videos.push_back(i);
    v.info.dims.push_back({i, 300, 340, 256});
  }
  for (uint32_t i = 0; i < n_videos; ++i) v.entries.push_back(&store.videos[i]);
  s.videos = v.info.videos.data();
  s.n_videos = n_videos;
  std::string why;
  if (sand::validate_spec(s, &why) != SAND_OK) {
    std::fprintf(stderr, "spec: %s\n", why.c_str());
    return 1;
  }
  sand::derive_spec(&v.info);
  double best = 1e30;
  size_t items = 0;
  std::shared_ptr<sand::EpochPlan> plan;
  for (int r = 0; r < reps; ++r) {
    const auto t0 = std::chrono::steady_clock::now();
    plan = sand::build_plan(v, (uint64_t)r, 0, std::move(plan));   // recycled, as the view does
    const auto t1 = std::chrono::steady_clock::now();
    best = std::min(best, std::chrono::duration<double, std::milli>(t1 - t0).count());
    items = plan->items.size();
  }
  std::printf("{\"config\": \"%s\", \"clips\": %u, \"items\": %zu, \"build_ms_best\": %.3f, \"us_per_clip\": %.3f}\n", cfg,
              n_videos, items, best, best * 1e3 / n_videos);
  return 0;
}
