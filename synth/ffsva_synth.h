/*
 * ffsva_synth.h — seeded synthetic surveillance video (WORKLOAD GENERATOR ONLY).
 *
 * This header is the one module shared by the CPU oracle's tests and the GPU
 * path's tests/benchmarks. It holds NONE of the method's arithmetic (no
 * downsampling, no distance, no threshold, no CNN): it only says what byte
 * value pixel (y, x, c) of frame t of stream s has, and which frames carry a
 * planted target object. It is compiled by gcc for the host generator
 * (synth_host.c) and by nvcc for the device generator (synth_cuda.cu); both
 * call exactly the same inline functions, so the two are byte-identical by
 * construction (tests/test_synth.py checks it on the GPU).
 *
 * Recipe, shaped like the paper's
 * workloads (Table 1: fixed-viewpoint 30-FPS surveillance
 * video; L123 Eq. (1) TOR; L177 target "scenes" of consecutive frames):
 *   background  B_s(y,x,c) = 64 + ((7(c+1)x + 5y + 16s) mod 96) + (h(bg,s,y>>4,x>>4,c) & 31)   in [64,190]
 *   noise       n = (h(noise,s,t,y,x,c) mod 5) - 2                                            (a = 2)
 *   pixel       B + n  (never clamps); inside the planted object: clamp(colour_c + n), colour_c in {0,255}
 *   schedule    period P frames, L_on consecutive target frames per period at phase h(phase,s) mod P
 *               (TOR = L_on / P exactly, Eq. (1))
 *   object      one rectangle, sides uniform in [ceil(W/8), W/5] x [ceil(H/8), H/5], moving linearly
 *               from a random start to a random end position over its scene, always fully inside
 *   reference   background frames use the independent noise tag "ref" ("average of
 *               dozens of background frames")
 * h() is splitmix64 chained over the key.
 */
#ifndef FFSVA_SYNTH_H
#define FFSVA_SYNTH_H

#include <stdint.h>

#if defined(__CUDACC__)
#define FFSVA_SYNTH_HD __host__ __device__ __forceinline__
#else
#define FFSVA_SYNTH_HD static inline
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef struct {
  uint64_t seed;
  int32_t  width, height;   /* raw frame size in pixels (RGB8 HWC) */
  int32_t  period;          /* P: schedule period in frames (300 in configs 1-4, 10 in config 5) */
  int32_t  on_len;          /* L_on: target frames per period (TOR * P) */
} ffsva_synth_params;

enum { FFSVA_TAG_BG = 1, FFSVA_TAG_NOISE = 2, FFSVA_TAG_REF = 3, FFSVA_TAG_OBJ = 4, FFSVA_TAG_PHASE = 5 };

FFSVA_SYNTH_HD uint64_t ffsva_sm64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

FFSVA_SYNTH_HD uint64_t ffsva_chain(uint64_t h, uint64_t k) {
  return ffsva_sm64(h ^ (k * 0xD1B54A32D192ED03ull));
}

/* Per-frame context: everything that does not depend on (y, x, c). */
typedef struct {
  uint64_t noise_key;
  uint64_t bg_key;
  int32_t  width, height, stream;
  int32_t  target;              /* 1 iff this frame carries the planted object */
  int32_t  ox, oy, ow, oh;      /* object rectangle [ox, ox+ow) x [oy, oy+oh) */
  int32_t  colour[3];           /* 0 or 255 per channel */
} ffsva_synth_ctx;

FFSVA_SYNTH_HD int32_t ffsva_synth_phase(const ffsva_synth_params* p, int32_t s) {
  return (int32_t)(ffsva_chain(ffsva_chain(p->seed, FFSVA_TAG_PHASE), (uint64_t)s) % (uint64_t)p->period);
}

/* 1 iff frame t of stream s is a planted target frame. */
FFSVA_SYNTH_HD int32_t ffsva_synth_is_target(const ffsva_synth_params* p, int32_t s, int64_t t) {
  int64_t u = t + p->period - ffsva_synth_phase(p, s);
  return (int32_t)((u % p->period) < p->on_len);
}

FFSVA_SYNTH_HD int32_t ffsva_synth_range(uint64_t h, int32_t lo, int32_t hi) {
  if (hi < lo) hi = lo;
  return lo + (int32_t)(h % (uint64_t)(hi - lo + 1));
}

/* Context of frame t of stream s (ref = 0), or of background reference frame t (ref = 1). */
FFSVA_SYNTH_HD void ffsva_synth_frame_ctx(const ffsva_synth_params* p, int32_t s, int64_t t, int32_t ref,
                                          ffsva_synth_ctx* c) {
  c->width = p->width;
  c->height = p->height;
  c->stream = s;
  c->bg_key = ffsva_chain(ffsva_chain(p->seed, FFSVA_TAG_BG), (uint64_t)s);
  c->noise_key = ffsva_chain(ffsva_chain(ffsva_chain(p->seed, ref ? FFSVA_TAG_REF : FFSVA_TAG_NOISE), (uint64_t)s),
                             (uint64_t)t);
  c->target = 0;
  c->ox = c->oy = c->ow = c->oh = 0;
  c->colour[0] = c->colour[1] = c->colour[2] = 0;
  if (ref || !ffsva_synth_is_target(p, s, t)) return;
  c->target = 1;
  {
    int64_t u = t + p->period - ffsva_synth_phase(p, s);
    int64_t scene = u / p->period;
    int32_t k = (int32_t)(u % p->period);
    uint64_t ho = ffsva_chain(ffsva_chain(ffsva_chain(p->seed, FFSVA_TAG_OBJ), (uint64_t)s), (uint64_t)scene);
    int32_t W = p->width, H = p->height;
    int32_t ow = ffsva_synth_range(ffsva_sm64(ho ^ 1), (W + 7) / 8, W / 5);
    int32_t oh = ffsva_synth_range(ffsva_sm64(ho ^ 2), (H + 7) / 8, H / 5);
    if (ow > W) ow = W;
    if (oh > H) oh = H;
    {
      int32_t xa = ffsva_synth_range(ffsva_sm64(ho ^ 3), 0, W - ow);
      int32_t xb = ffsva_synth_range(ffsva_sm64(ho ^ 4), 0, W - ow);
      int32_t ya = ffsva_synth_range(ffsva_sm64(ho ^ 5), 0, H - oh);
      int32_t yb = ffsva_synth_range(ffsva_sm64(ho ^ 6), 0, H - oh);
      int32_t den = p->on_len > 1 ? p->on_len - 1 : 1;
      uint64_t hc = ffsva_sm64(ho ^ 7);
      c->ox = xa + (int32_t)(((int64_t)(xb - xa) * k) / den);
      c->oy = ya + (int32_t)(((int64_t)(yb - ya) * k) / den);
      c->ow = ow;
      c->oh = oh;
      c->colour[0] = (hc & 1) ? 255 : 0;
      c->colour[1] = (hc & 2) ? 255 : 0;
      c->colour[2] = (hc & 4) ? 255 : 0;
    }
  }
}

FFSVA_SYNTH_HD int32_t ffsva_synth_background(const ffsva_synth_ctx* c, int32_t y, int32_t x, int32_t ch) {
  uint64_t cell = ((((uint64_t)(y >> 4)) << 20) | (uint64_t)(x >> 4)) * 4u + (uint64_t)ch;
  return 64 + ((7 * (ch + 1) * x + 5 * y + 16 * c->stream) % 96) + (int32_t)(ffsva_chain(c->bg_key, cell) & 31u);
}

FFSVA_SYNTH_HD uint8_t ffsva_synth_pixel(const ffsva_synth_ctx* c, int32_t y, int32_t x, int32_t ch) {
  uint64_t idx = ((uint64_t)y * (uint64_t)c->width + (uint64_t)x) * 3u + (uint64_t)ch;
  int32_t n = (int32_t)(ffsva_sm64(c->noise_key ^ idx) % 5u) - 2;
  int32_t v;
  if (c->target && x >= c->ox && x < c->ox + c->ow && y >= c->oy && y < c->oy + c->oh) {
    v = c->colour[ch] + n;
    v = v < 0 ? 0 : (v > 255 ? 255 : v);
  } else {
    v = ffsva_synth_background(c, y, x, ch) + n;
  }
  return (uint8_t)v;
}

#ifdef __cplusplus
}
#endif

#endif /* FFSVA_SYNTH_H */
