// planner.h — host-side epoch planner of the product.
//
// Independent implementation of the sampling definitions (R#1-R#18): it
// shares no code with oracle/ (DESIGN.md §4). Everything here is integer or IEEE
// double arithmetic with glibc transcendentals, compiled with -ffp-contract=off,
// so the draws are bit-identical to the oracle's by construction of the readings
// (checked bit-exactly by tests/test_gpu_parity.py via sand_view_get_meta).
#pragma once
#include <array>
#include <cstdint>
#include <string>
#include <vector>

#include "sand.h"

namespace sand {

// Counter-based generator: Philox4x32-10 keyed by the 64-bit seed (R#1).
class Philox4x32 {
 public:
  explicit Philox4x32(uint64_t seed) : k0_(static_cast<uint32_t>(seed)), k1_(static_cast<uint32_t>(seed >> 32)) {}
  std::array<uint32_t, 4> operator()(std::array<uint32_t, 4> ctr) const;

 private:
  uint32_t k0_, k1_;
};

enum class Purpose : uint32_t { kPerm = 1, kTemporal = 2, kCrop = 3, kAug = 4, kWindow = 5 };

// The draws of one epoch: counter (index, purpose<<24|group<<16|sub, unit, epoch lo); the epoch's
// high 32 bits are XORed into the key's high word (R#1), so epochs e and e + 2^32 draw
// independent streams while every epoch below 2^32 keeps the plain (seed lo, seed hi) key.
class EpochDraws {
 public:
  EpochDraws(uint64_t seed, uint64_t epoch)
      : gen_(seed ^ (epoch & 0xffffffff00000000ull)), epoch_lo_(static_cast<uint32_t>(epoch)) {}
  std::array<uint32_t, 4> get(Purpose p, uint32_t group, uint32_t sub, uint32_t index, uint32_t unit) const {
    const uint32_t tag = (static_cast<uint32_t>(p) << 24) | ((group & 0xffu) << 16) | (sub & 0xffffu);
    return gen_({index, tag, unit, epoch_lo_});
  }

 private:
  Philox4x32 gen_;
  uint32_t epoch_lo_;
};

inline uint32_t draw_below(uint32_t x, uint32_t n) {          // Lemire multiply-shift
  return static_cast<uint32_t>((static_cast<uint64_t>(x) * n) >> 32);
}
inline double draw_unit(uint32_t x) { return static_cast<double>(x) / 4294967296.0; }
bool draw_coin(uint32_t x, double p);

struct VideoDims {
  uint32_t id, n_frames, width, height;
};

// Owned copy of a sand_view_spec plus derived, per-group information.
struct SpecInfo {
  sand_view_spec spec{};
  std::vector<uint32_t> videos;      // dataset order
  std::vector<VideoDims> dims;       // parallel to videos
  int leader[SAND_MAX_GROUPS] = {-1, -1, -1, -1, -1, -1, -1, -1};  // lowest view index per group
  std::vector<uint32_t> groups;      // group ids in use, increasing
  uint32_t g = 1, pool_len = 1;      // gcd of strides; pool length L in grid points
  uint32_t span[SAND_MAX_VIEWS] = {};
};

// Validate a spec; on success fill `info` (dims resolved by the caller). Returns
// SAND_OK or SAND_EINVAL with a message in `why`.
int validate_spec(const sand_view_spec& spec, std::string* why);
void derive_spec(SpecInfo* info);

// DistributedSampler partition of the permuted clip list for one rank (R#2, R#3).
uint32_t samples_per_rank(uint32_t n_clips, uint32_t world, bool drop_last);
std::vector<uint32_t> rank_clips(const SpecInfo& info, uint64_t epoch, uint32_t rank);

// Temporal + spatial plan of one clip (R#4-R#18), written as a sand_clip_meta.
void plan_clip(const SpecInfo& info, uint64_t epoch, uint32_t clip, sand_clip_meta* meta);

}  // namespace sand
