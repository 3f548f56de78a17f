/*
 * synth_host.c — host (CPU) twin of the synthetic video generator.
 * Workload generation only; see ffsva_synth.h for the recipe. Built into
 * synth/libffsva_synth.so by __graft_entry__.build().
 */
#include "ffsva_synth.h"

/* Write frame t of stream s (ref = 0) or background reference frame t (ref = 1)
 * as H rows of 3*W bytes, rows `pitch` bytes apart. */
void ffsva_synth_frame(const ffsva_synth_params* p, int32_t s, int64_t t, int32_t ref, uint8_t* out, int64_t pitch) {
  ffsva_synth_ctx c;
  ffsva_synth_frame_ctx(p, s, t, ref, &c);
  for (int32_t y = 0; y < p->height; ++y) {
    uint8_t* row = out + (int64_t)y * pitch;
    for (int32_t x = 0; x < p->width; ++x)
      for (int32_t ch = 0; ch < 3; ++ch) row[3 * x + ch] = ffsva_synth_pixel(&c, y, x, ch);
  }
}

/* n frames (streams[i], frames[i]) into out + i*frame_stride. */
void ffsva_synth_frames(const ffsva_synth_params* p, const int32_t* streams, const int64_t* frames, int32_t n,
                        int32_t ref, uint8_t* out, int64_t frame_stride, int64_t pitch) {
  for (int32_t i = 0; i < n; ++i) ffsva_synth_frame(p, streams[i], frames[i], ref, out + (int64_t)i * frame_stride, pitch);
}

int32_t ffsva_synth_target(const ffsva_synth_params* p, int32_t s, int64_t t) { return ffsva_synth_is_target(p, s, t); }

/* Number of planted target frames of stream s in [t0, t1). */
int64_t ffsva_synth_planted(const ffsva_synth_params* p, int32_t s, int64_t t0, int64_t t1) {
  int64_t n = 0;
  for (int64_t t = t0; t < t1; ++t) n += ffsva_synth_is_target(p, s, t);
  return n;
}

/* Object rectangle of frame t of stream s: out[0..3] = ox, oy, ow, oh (all 0 if not a target frame). */
void ffsva_synth_object(const ffsva_synth_params* p, int32_t s, int64_t t, int32_t* out) {
  ffsva_synth_ctx c;
  ffsva_synth_frame_ctx(p, s, t, 0, &c);
  out[0] = c.ox;
  out[1] = c.oy;
  out[2] = c.ow;
  out[3] = c.oh;
}
