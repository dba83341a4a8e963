/*
 * nv12_synth.h — seeded, counter-based synthetic NV12 frame generator.
 *
 * This module is the ONLY code shared between the CUDA product path and the
 * CPU oracle (DESIGN.md §3 "input recipe"). It holds none of the method's
 * arithmetic: it only decides the bytes of the synthetic "decoded" frames that
 * stand in for decoder output (BASELINE.json north_star: "synthetic raw NV12
 * frames stand in for decoder output"). Every byte is a pure function of
 * (seed, video, frame, plane, row, column), so the host generator (oracle side)
 * and the device generator (store fill) are bit-identical by construction.
 *
 * NV12 layout of one W x H frame (W, H even):
 *   plane 0 (Y):  H rows of W bytes
 *   plane 1 (UV): H/2 rows of W bytes, interleaved U,V per 2x2 luma block
 *
 * Families:
 *   SYNTH_UNIFORM : i.i.d.-looking uniform bytes (throughput default; worst case
 *                   for RGB gamut clamping)
 *   SYNTH_SMOOTH  : legal-range (Y 16..235, UV 16..240) integer triangle waves
 *                   drifting with the frame index (natural-video-like motion)
 */
#ifndef SYNTH_NV12_SYNTH_H
#define SYNTH_NV12_SYNTH_H

#include <stdint.h>

#if defined(__CUDACC__)
#define SYNTH_FN __host__ __device__ __forceinline__ static
#else
#define SYNTH_FN static inline
#endif

enum { SYNTH_UNIFORM = 0, SYNTH_SMOOTH = 1 };

/* murmur3 32-bit finaliser */
SYNTH_FN uint32_t synth_fmix32(uint32_t h) {
  h ^= h >> 16;
  h *= 0x85ebca6bu;
  h ^= h >> 13;
  h *= 0xc2b2ae35u;
  h ^= h >> 16;
  return h;
}

/* Hash prefix for one (seed, video, frame, plane, row). */
SYNTH_FN uint32_t synth_row_key(uint64_t seed, uint32_t video, uint32_t frame,
                                uint32_t plane, uint32_t row) {
  uint32_t h = synth_fmix32((uint32_t)seed ^ 0x9e3779b9u);
  h = synth_fmix32(h ^ (uint32_t)(seed >> 32) ^ 0x7f4a7c15u);
  h = synth_fmix32(h + video * 0x85ebca77u);
  h = synth_fmix32(h + frame * 0xc2b2ae3du + plane);
  h = synth_fmix32(h + row * 0x27d4eb2fu);
  return h;
}

/* 4 consecutive bytes [4*q, 4*q+3] of a row, little-endian packed. */
SYNTH_FN uint32_t synth_uniform_word(uint32_t row_key, uint32_t q) {
  return synth_fmix32(row_key ^ (q * 0x165667b1u + 0x9e3779b9u));
}

SYNTH_FN uint32_t synth_tri(uint32_t p, uint32_t half) { /* 0..half-1..0 */
  return p < half ? p : 2u * half - 1u - p;
}

/* One byte of the SMOOTH family. plane 0: Y in [16,235]; plane 1: U/V in [16,240]. */
SYNTH_FN uint8_t synth_smooth_byte(uint64_t seed, uint32_t video, uint32_t frame,
                                   uint32_t plane, uint32_t row, uint32_t col) {
  uint32_t s = (uint32_t)seed * 7u + video * 13u;
  if (plane == 0) {
    uint32_t p = (col * 3u + row * 2u + frame * 5u + s) % 440u;
    return (uint8_t)(16u + synth_tri(p, 220u));
  } else {
    uint32_t isv = col & 1u;
    uint32_t p = ((col >> 1) * 5u + row * 3u + frame * 2u + s + isv * 101u) % 450u;
    return (uint8_t)(16u + synth_tri(p, 225u));
  }
}

/* Byte at (plane, row, col) of frame (video, frame) for the given family. */
SYNTH_FN uint8_t synth_byte(int family, uint64_t seed, uint32_t video, uint32_t frame,
                            uint32_t plane, uint32_t row, uint32_t col) {
  if (family == SYNTH_SMOOTH) return synth_smooth_byte(seed, video, frame, plane, row, col);
  uint32_t w = synth_uniform_word(synth_row_key(seed, video, frame, plane, row), col >> 2);
  return (uint8_t)(w >> (8u * (col & 3u)));
}

#endif /* SYNTH_NV12_SYNTH_H */
