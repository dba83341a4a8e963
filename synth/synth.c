/*
 * synth.c — host side of the synthetic NV12 generator (see nv12_synth.h).
 * Built into libsynth_host.so; used by tests, the oracle harness and bench.py to
 * produce the same bytes the device generator (synth_cuda.cu) writes.
 */
#include <stddef.h>
#include <stdint.h>
#include "nv12_synth.h"

/* Fill n_frames consecutive frames of one video. y/uv point at the first frame;
 * consecutive frames are frame_stride bytes apart in both buffers. */
int synth_fill_frames(int family, uint64_t seed, uint32_t video, uint32_t first_frame,
                      uint32_t n_frames, uint32_t width, uint32_t height,
                      uint8_t* y, size_t y_pitch, uint8_t* uv, size_t uv_pitch,
                      size_t frame_stride) {
  if ((width & 1u) || (height & 1u) || width == 0 || height == 0) return -1;
  for (uint32_t f = 0; f < n_frames; ++f) {
    uint32_t frame = first_frame + f;
    uint8_t* yf = y + (size_t)f * frame_stride;
    uint8_t* uvf = uv + (size_t)f * frame_stride;
    for (uint32_t plane = 0; plane < 2; ++plane) {
      uint32_t rows = plane == 0 ? height : height / 2;
      uint8_t* base = plane == 0 ? yf : uvf;
      size_t pitch = plane == 0 ? y_pitch : uv_pitch;
      for (uint32_t r = 0; r < rows; ++r) {
        uint8_t* row = base + (size_t)r * pitch;
        if (family == SYNTH_SMOOTH) {
          for (uint32_t c = 0; c < width; ++c)
            row[c] = synth_smooth_byte(seed, video, frame, plane, r, c);
        } else {
          uint32_t key = synth_row_key(seed, video, frame, plane, r);
          for (uint32_t c = 0; c < width; c += 4) {
            uint32_t w = synth_uniform_word(key, c >> 2);
            for (uint32_t k = 0; k < 4 && c + k < width; ++k) row[c + k] = (uint8_t)(w >> (8 * k));
          }
        }
      }
    }
  }
  return 0;
}
