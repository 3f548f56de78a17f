/*
 * ffsva_oracle.c — CPU ORACLE for the FFS-VA SDD + SNM filter cascade.
 *
 * TEST INFRASTRUCTURE ONLY (see ffsva_oracle.h): only tests/,
 * __graft_entry__.smoke() and bench.py's CPU-baseline leg use it. Plain,
 * slow, single-threaded definitions, each citing the PAPER.md passage it
 * follows. Shares no code with the CUDA path.
 */
#include "ffsva_oracle.h"

#include <math.h>
#include <stdlib.h>
#include <string.h>

/* Cell i of a dimension of S samples split into D cells covers [floor(i*S/D), floor((i+1)*S/D)). */
static int64_t cell_lo(int64_t i, int64_t S, int64_t D) { return (i * S) / D; }

/* PAPER.md L187 (resize before each filter), L155 (SDD 100x100), L167 (SNM 50x50); SURVEY §8(c) C1. */
void orc_box_downsample(const uint8_t* frame, int32_t W, int32_t H, int64_t pitch, int32_t Dw, int32_t Dh,
                        uint8_t* out) {
  for (int32_t oy = 0; oy < Dh; ++oy) {
    int64_t y0 = cell_lo(oy, H, Dh), y1 = cell_lo(oy + 1, H, Dh);
    for (int32_t ox = 0; ox < Dw; ++ox) {
      int64_t x0 = cell_lo(ox, W, Dw), x1 = cell_lo(ox + 1, W, Dw);
      int64_t n = (y1 - y0) * (x1 - x0);
      for (int32_t c = 0; c < 3; ++c) {
        int64_t s = 0;
        for (int64_t y = y0; y < y1; ++y)
          for (int64_t x = x0; x < x1; ++x) s += frame[y * pitch + 3 * x + c];
        out[((int64_t)oy * Dw + ox) * 3 + c] = (uint8_t)((s + n / 2) / n);
      }
    }
  }
}

/* "the reference image is usually computed as the average of dozens of background frames".
 * single rounding of the mean over the K frames x box samples. */
void orc_reference(const uint8_t* frames, int32_t K, int64_t frame_stride, int32_t W, int32_t H, int64_t pitch,
                   int32_t Dw, int32_t Dh, uint8_t* out) {
  for (int32_t oy = 0; oy < Dh; ++oy) {
    int64_t y0 = cell_lo(oy, H, Dh), y1 = cell_lo(oy + 1, H, Dh);
    for (int32_t ox = 0; ox < Dw; ++ox) {
      int64_t x0 = cell_lo(ox, W, Dw), x1 = cell_lo(ox + 1, W, Dw);
      int64_t n = (int64_t)K * (y1 - y0) * (x1 - x0);
      for (int32_t c = 0; c < 3; ++c) {
        int64_t s = 0;
        for (int32_t k = 0; k < K; ++k)
          for (int64_t y = y0; y < y1; ++y)
            for (int64_t x = x0; x < x1; ++x) s += frames[k * frame_stride + y * pitch + 3 * x + c];
        out[((int64_t)oy * Dw + ox) * 3 + c] = (uint8_t)((s + n / 2) / n);
      }
    }
  }
}

/* distance by MSE ("Take MSE as an example"); SSD = N * MSE kept exact in u64. */
uint64_t orc_ssd(const uint8_t* a, const uint8_t* b, int64_t N) {
  uint64_t s = 0;
  for (int64_t i = 0; i < N; ++i) {
    int64_t d = (int64_t)a[i] - (int64_t)b[i];
    s += (uint64_t)(d * d);
  }
  return s;
}

/* "if MSE is larger than the threshold delta_diff, an obvious content change is construed".
 * MSE > delta  <=>  SSD > delta*N  <=>  SSD > floor(delta*N) for integer SSD, with delta*N taken EXACTLY
 * (a rounded double product can land on the integer just above the true value, e.g. delta = 1/3 in double,
 * N = 30000). delta = m * 2^(e-53) with integer m, so delta*N = (m*N) * 2^(e-53) is exact in 128 bits. */
uint64_t orc_threshold(double delta_diff, int64_t N) {
  if (!(delta_diff > 0.0) || N <= 0) return 0;
  int e;
  double f = frexp(delta_diff, &e);                 /* delta = f * 2^e, f in [0.5, 1) */
  unsigned __int128 m = (unsigned __int128)ldexp(f, 53); /* exact 53-bit integer */
  unsigned __int128 q = m * (unsigned __int128)N;
  int sh = e - 53;
  if (sh >= 0) {
    if (sh >= 64 || (q << sh) >> sh != q || (q << sh) > (unsigned __int128)UINT64_MAX) return UINT64_MAX;
    return (uint64_t)(q << sh);
  }
  if (-sh >= 128) return 0;
  q >>= -sh;                                          /* floor, q >= 0 */
  return q > (unsigned __int128)UINT64_MAX ? UINT64_MAX : (uint64_t)q;
}

int32_t orc_sdd_pass(uint64_t ssd, uint64_t T) { return ssd > T ? 1 : 0; }

/* "The distance between two video frames can be characterized by ... Sum of Absolute
 * Differences (SAD)". SAD = sum |a - b| over the N values, in u64 (reading Q23: pass iff
 * SAD > delta_diff, i.e. SAD > floor(delta_diff) = orc_threshold(delta_diff, 1)). */
uint64_t orc_sad(const uint8_t* a, const uint8_t* b, int64_t N) {
  uint64_t s = 0;
  for (int64_t i = 0; i < N; ++i) {
    int64_t d = (int64_t)a[i] - (int64_t)b[i];
    s += (uint64_t)(d < 0 ? -d : d);
  }
  return s;
}

/* PAPER.md L151 NRMSE (reading Q24: Euclidean normalisation, NRMSE = sqrt(SSD / sum R^2)):
 * the normaliser sum of squares of the reference image, in u64. */
uint64_t orc_sum_sq(const uint8_t* a, int64_t N) {
  uint64_t s = 0;
  for (int64_t i = 0; i < N; ++i) s += (uint64_t)a[i] * (uint64_t)a[i];
  return s;
}

/* SDD survivors are pushed to the SNM queue in arrival order. */
int32_t orc_compact(const uint8_t* pass, int32_t n, int32_t* idx) {
  int32_t m = 0;
  for (int32_t i = 0; i < n; ++i)
    if (pass[i]) idx[m++] = i;
  return m;
}

/* Round to 8 significant bits, ties to even (nearbyint under the default FE_TONEAREST mode). */
double orc_round_bf16(double x) {
  if (x == 0.0 || !isfinite(x)) return x;
  int e;
  double m = frexp(x, &e); /* x = m * 2^e, |m| in [0.5, 1) */
  return ldexp(nearbyint(ldexp(m, 8)), e - 8);
}

/* PAPER.md L159 CONV layer; cross-correlation, zero padding 1, stride 1. */
void orc_conv3x3(const double* in, int32_t C, int32_t H, int32_t W, const double* w, const double* b, int32_t K,
                 double* out) {
  for (int32_t k = 0; k < K; ++k)
    for (int32_t y = 0; y < H; ++y)
      for (int32_t x = 0; x < W; ++x) {
        double s = b ? b[k] : 0.0;
        for (int32_t c = 0; c < C; ++c)
          for (int32_t dy = 0; dy < 3; ++dy)
            for (int32_t dx = 0; dx < 3; ++dx) {
              int32_t yy = y + dy - 1, xx = x + dx - 1;
              if (yy < 0 || yy >= H || xx < 0 || xx >= W) continue;
              s += in[((int64_t)c * H + yy) * W + xx] * w[(((int64_t)k * C + c) * 3 + dy) * 3 + dx];
            }
        out[((int64_t)k * H + y) * W + x] = s;
      }
}

/* 2x2 max-pool, stride 2, floor: out is C x floor(H/2) x floor(W/2). */
void orc_maxpool2(const double* in, int32_t C, int32_t H, int32_t W, double* out) {
  int32_t Ho = H / 2, Wo = W / 2;
  for (int32_t c = 0; c < C; ++c)
    for (int32_t y = 0; y < Ho; ++y)
      for (int32_t x = 0; x < Wo; ++x) {
        double m = in[((int64_t)c * H + 2 * y) * W + 2 * x];
        for (int32_t dy = 0; dy < 2; ++dy)
          for (int32_t dx = 0; dx < 2; ++dx) {
            double v = in[((int64_t)c * H + 2 * y + dy) * W + 2 * x + dx];
            if (v > m) m = v;
          }
        out[((int64_t)c * Ho + y) * Wo + x] = m;
      }
}

static void relu_inplace(double* v, int64_t n) {
  for (int64_t i = 0; i < n; ++i)
    if (v[i] < 0.0) v[i] = 0.0;
}

int64_t orc_snm_n_params(int32_t h, int32_t w, int32_t c1, int32_t c2) {
  int64_t F = (int64_t)c2 * ((h / 2) / 2) * ((w / 2) / 2);
  return 27LL * c1 + c1 + 9LL * c1 * c2 + c2 + F + 1;
}

/* "SNM is a three-layer CNN (CONV, CONV, and FC)" that "outputs a predicted probability c";
 * L167: 50x50 input. Topology and precision readings: SURVEY §8(c) C5, C6, Q9-Q11, Q15. */
double orc_snm_forward(const uint8_t* d50, int32_t h, int32_t w, const float* params, int32_t c1, int32_t c2,
                       int32_t bf16_emul) {
  int32_t h1 = h / 2, w1s = w / 2, h2 = h1 / 2, w2s = w1s / 2;
  int64_t F = (int64_t)c2 * h2 * w2s;
  const float* pw1 = params;
  const float* pb1 = pw1 + 27 * c1;
  const float* pw2 = pb1 + c1;
  const float* pb2 = pw2 + 9 * c1 * c2;
  const float* pwfc = pb2 + c2;
  const float* pbfc = pwfc + F;

  double* x = malloc(sizeof(double) * 3 * h * w);
  double* wt1 = malloc(sizeof(double) * 27 * c1);
  double* bb1 = malloc(sizeof(double) * c1);
  double* wt2 = malloc(sizeof(double) * 9 * c1 * c2);
  double* bb2 = malloc(sizeof(double) * c2);
  double* a1 = malloc(sizeof(double) * c1 * h * w);
  double* p1 = malloc(sizeof(double) * c1 * h1 * w1s);
  double* a2 = malloc(sizeof(double) * c2 * h1 * w1s);
  double* p2 = malloc(sizeof(double) * F);

  /* C5: x[c][y][x] = (D50[y][x][c] - 128) / 128 */
  for (int32_t c = 0; c < 3; ++c)
    for (int32_t y = 0; y < h; ++y)
      for (int32_t xx = 0; xx < w; ++xx) x[((int64_t)c * h + y) * w + xx] = ((double)d50[((int64_t)y * w + xx) * 3 + c] - 128.0) / 128.0;
  for (int32_t i = 0; i < 27 * c1; ++i) wt1[i] = bf16_emul ? orc_round_bf16(pw1[i]) : (double)pw1[i];
  for (int32_t i = 0; i < c1; ++i) bb1[i] = pb1[i];
  for (int32_t i = 0; i < 9 * c1 * c2; ++i) wt2[i] = bf16_emul ? orc_round_bf16(pw2[i]) : (double)pw2[i];
  for (int32_t i = 0; i < c2; ++i) bb2[i] = pb2[i];

  /* CONV 1 -> ReLU -> max-pool */
  orc_conv3x3(x, 3, h, w, wt1, bb1, c1, a1);
  relu_inplace(a1, (int64_t)c1 * h * w);
  orc_maxpool2(a1, c1, h, w, p1);
  if (bf16_emul)
    for (int64_t i = 0; i < (int64_t)c1 * h1 * w1s; ++i) p1[i] = orc_round_bf16(p1[i]);
  /* CONV 2 -> ReLU -> max-pool */
  orc_conv3x3(p1, c1, h1, w1s, wt2, bb2, c2, a2);
  relu_inplace(a2, (int64_t)c2 * h1 * w1s);
  orc_maxpool2(a2, c2, h1, w1s, p2);
  /* FC over the CHW-flattened features -> one logit */
  double logit = (double)pbfc[0];
  for (int64_t i = 0; i < F; ++i) logit += (bf16_emul ? orc_round_bf16(pwfc[i]) : (double)pwfc[i]) * p2[i];

  free(x); free(wt1); free(bb1); free(wt2); free(bb2); free(a1); free(p1); free(a2); free(p2);
  return logit;
}

/* PAPER.md L193 Eq. (2): t_pre = (c_high - c_low) * FilterDegree + c_low. */
double orc_tpre(double c_low, double c_high, double filter_degree) {
  return (c_high - c_low) * filter_degree + c_low;
}

double orc_logit(double t) {
  if (t <= 0.0) return -INFINITY;
  if (t >= 1.0) return INFINITY;
  return log(t / (1.0 - t));
}

/* PAPER.md L159 (c < c_low: no target; c > c_high: target; otherwise unsure) and L165 (c >= t_pre goes on,
 * c < t_pre is filtered out). c = sigmoid(logit) is strictly increasing, so each test is done on the logit. */
void orc_decide(double logit, double c_low, double c_high, double filter_degree, uint8_t* pass, uint8_t* cls) {
  double lt = orc_logit(orc_tpre(c_low, c_high, filter_degree));
  *pass = logit >= lt ? 1 : 0;
  if (logit < orc_logit(c_low)) *cls = 0;
  else if (logit > orc_logit(c_high)) *cls = 2;
  else *cls = 1;
}

/* ===================================================================================== f1: T-YOLO (L169-L175) */

/* Q28: cell i covers [floor(iS/D), max(floor((i+1)S/D), floor(iS/D) + 1)). */
void orc_resize(const uint8_t* frame, int32_t W, int32_t H, int64_t pitch, int32_t Dw, int32_t Dh, uint8_t* out) {
  for (int32_t oy = 0; oy < Dh; ++oy) {
    int64_t y0 = cell_lo(oy, H, Dh), y1 = cell_lo(oy + 1, H, Dh);
    if (y1 <= y0) y1 = y0 + 1;
    for (int32_t ox = 0; ox < Dw; ++ox) {
      int64_t x0 = cell_lo(ox, W, Dw), x1 = cell_lo(ox + 1, W, Dw);
      if (x1 <= x0) x1 = x0 + 1;
      int64_t n = (y1 - y0) * (x1 - x0);
      for (int32_t c = 0; c < 3; ++c) {
        int64_t sum = 0;
        for (int64_t y = y0; y < y1; ++y)
          for (int64_t x = x0; x < x1; ++x) sum += frame[y * pitch + 3 * x + c];
        out[((int64_t)oy * Dw + ox) * 3 + c] = (uint8_t)((sum + n / 2) / n);
      }
    }
  }
}

void orc_conv1x1(const double* in, int32_t C, int32_t H, int32_t W, const double* w, const double* b, int32_t K,
                 double* out) {
  for (int32_t k = 0; k < K; ++k)
    for (int64_t p = 0; p < (int64_t)H * W; ++p) {
      double s = b ? b[k] : 0.0;
      for (int32_t c = 0; c < C; ++c) s += in[(int64_t)c * H * W + p] * w[(int64_t)k * C + c];
      out[(int64_t)k * H * W + p] = s;
    }
}

void orc_leaky(double* v, int64_t n) {
  for (int64_t i = 0; i < n; ++i)
    if (v[i] < 0.0) v[i] *= 0.1;
}

void orc_maxpool2_s1(const double* in, int32_t C, int32_t H, int32_t W, double* out) {
  for (int32_t c = 0; c < C; ++c)
    for (int32_t y = 0; y < H; ++y)
      for (int32_t x = 0; x < W; ++x) {
        double m = in[((int64_t)c * H + y) * W + x];
        for (int32_t dy = 0; dy < 2; ++dy)
          for (int32_t dx = 0; dx < 2; ++dx) {
            if (y + dy >= H || x + dx >= W) continue;
            double v = in[((int64_t)c * H + y + dy) * W + x + dx];
            if (v > m) m = v;
          }
        out[((int64_t)c * H + y) * W + x] = m;
      }
}

/* tiny-yolo-voc topology: (Cin, Cout, kernel, pool after: 0 none, 1 = 2x2/2, 2 = 2x2/1) */
static const int32_t kTyolo[9][4] = {{3, 16, 3, 1},     {16, 32, 3, 1},     {32, 64, 3, 1},
                                     {64, 128, 3, 1},   {128, 256, 3, 1},   {256, 512, 3, 2},
                                     {512, 1024, 3, 0}, {1024, 1024, 3, 0}, {1024, 125, 1, 0}};

int64_t orc_tyolo_n_params(void) {
  int64_t n = 0;
  for (int l = 0; l < 9; ++l) n += (int64_t)kTyolo[l][1] * kTyolo[l][0] * kTyolo[l][2] * kTyolo[l][2] + kTyolo[l][1];
  return n;
}

/* 9 CONV + 6 POOL layers on 416x416 input; L171: 13x13 grid x 5 boxes. */
int32_t orc_tyolo_forward(const uint8_t* img, int32_t S, const float* params, int32_t bf16_emul, double* out) {
  if (S <= 0 || S % 32) return -1;
  int32_t H = S, W = S;
  double* x = malloc(sizeof(double) * 3 * (size_t)S * S);
  for (int32_t c = 0; c < 3; ++c) /* Q29: x = v / 256, CHW */
    for (int64_t p = 0; p < (int64_t)S * S; ++p) x[(int64_t)c * S * S + p] = (double)img[p * 3 + c] / 256.0;
  const float* pp = params;
  for (int l = 0; l < 9; ++l) {
    const int32_t C = kTyolo[l][0], K = kTyolo[l][1], k = kTyolo[l][2], pool = kTyolo[l][3];
    const int64_t nw = (int64_t)K * C * k * k;
    double* w = malloc(sizeof(double) * nw);
    double* b = malloc(sizeof(double) * K);
    for (int64_t i = 0; i < nw; ++i) w[i] = bf16_emul ? orc_round_bf16(pp[i]) : (double)pp[i];
    for (int32_t i = 0; i < K; ++i) b[i] = pp[nw + i];
    pp += nw + K;
    double* y = malloc(sizeof(double) * K * (size_t)H * W);
    if (k == 3)
      orc_conv3x3(x, C, H, W, w, b, K, y);
    else
      orc_conv1x1(x, C, H, W, w, b, K, y);
    if (l < 8) orc_leaky(y, (int64_t)K * H * W);
    free(x);
    free(w);
    free(b);
    if (pool == 1) {
      double* z = malloc(sizeof(double) * K * (size_t)(H / 2) * (W / 2));
      orc_maxpool2(y, K, H, W, z);
      free(y);
      y = z;
      H /= 2;
      W /= 2;
    } else if (pool == 2) {
      double* z = malloc(sizeof(double) * K * (size_t)H * W);
      orc_maxpool2_s1(y, K, H, W, z);
      free(y);
      y = z;
    }
    if (bf16_emul && l < 8)
      for (int64_t i = 0; i < (int64_t)K * H * W; ++i) y[i] = orc_round_bf16(y[i]);
    x = y;
  }
  /* CHW -> HWC */
  for (int32_t c = 0; c < 125; ++c)
    for (int64_t p = 0; p < (int64_t)H * W; ++p) out[p * 125 + c] = x[(int64_t)c * H * W + p];
  free(x);
  return 0;
}

/* L171 "If the confidence score exceeds the threshold (e.g., 0.2), one target object is considered to appear";
 * L195 NumberofObjects. Confidence of box b = sigmoid(objectness) * softmax(class logits)[target] (Q31). */
int32_t orc_tyolo_count(const double* out, int32_t cells, int32_t target_class, double thresh) {
  int32_t n = 0;
  for (int32_t p = 0; p < cells; ++p)
    for (int32_t b = 0; b < 5; ++b) {
      const double* v = out + (int64_t)p * 125 + 25 * b;
      double mx = v[5];
      for (int32_t k = 1; k < 20; ++k)
        if (v[5 + k] > mx) mx = v[5 + k];
      double z = 0.0;
      for (int32_t k = 0; k < 20; ++k) z += exp(v[5 + k] - mx);
      const double score = 1.0 / (1.0 + exp(-v[4])) * exp(v[5 + target_class] - mx) / z;
      if (score > thresh) ++n;
    }
  return n;
}
