/*
 * ffsva_oracle.h — CPU ORACLE for the FFS-VA SDD + SNM filter cascade.
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference leg may load or call this. The
 * product (paper_conf_icpp_zhangcjzly18_b200/, include/ffsva.h) never does;
 * the two share no code, headers, tables or helpers.
 *
 * Every function is the plain definition of what the paper's step computes
 * (PAPER.md line numbers; readings from SURVEY.md §8(c) C1-C8 / Q1-Q22, listed
 * in DESIGN.md "Readings"). Single-threaded loop nests, no SIMD, no blocking,
 * no fusion; fp64 for floating point (the paper fixes no precision).
 * Every function is pinned by tests/test_oracle.py (pins P1-P12); none is
 * "parity unpinned".
 */
#ifndef FFSVA_ORACLE_H
#define FFSVA_ORACLE_H
#include <stdint.h>

/* C1 ("raw frames need to be resized to meet the filter's feature size"; Q1/Q2):
 * integer box average of an H x W RGB8 frame (rows `pitch` bytes apart) onto a Dh x Dw grid.
 * Cell i of a source dimension S covers [floor(i*S/D), floor((i+1)*S/D)); value = (s + n/2) / n. */
void orc_box_downsample(const uint8_t* frame, int32_t W, int32_t H, int64_t pitch, int32_t Dw, int32_t Dh,
                        uint8_t* out);

/* C2 ("the reference image is usually computed as the average of dozens of background
 * frames"; Q6): one rounding of the mean over all K*n samples of each cell. */
void orc_reference(const uint8_t* frames, int32_t K, int64_t frame_stride, int32_t W, int32_t H, int64_t pitch,
                   int32_t Dw, int32_t Dh, uint8_t* out);

/* C3 (PAPER.md L151 MSE; Q4): SSD = sum (a - b)^2 over N values, in u64. MSE = SSD / N. */
uint64_t orc_ssd(const uint8_t* a, const uint8_t* b, int64_t N);

/* C3 ("if MSE is larger than the threshold delta_diff"; Q5): T = floor(delta * N) with the
 * product taken exactly (not rounded in double); pass iff SSD > T, i.e. iff SSD/N > delta exactly. */
uint64_t orc_threshold(double delta_diff, int64_t N);
int32_t orc_sdd_pass(uint64_t ssd, uint64_t T);

/* f3 SDD variants ("MSE, NRMSE, or SAD"; readings Q23, Q24):
 * SAD = sum |a - b| (u64); pass iff SAD > floor(delta_diff).
 * NRMSE = sqrt(SSD / sum R^2); pass iff NRMSE > delta_diff <=> SSD > floor(delta_diff^2 * sum R^2), the product
 * taken exactly (oracle.nrmse_threshold, Python fractions). */
uint64_t orc_sad(const uint8_t* a, const uint8_t* b, int64_t N);
uint64_t orc_sum_sq(const uint8_t* a, int64_t N);

/* C4 (PAPER.md L143 survivors forwarded in order; Q16): idx[0..m) = passing indices in batch order. */
int32_t orc_compact(const uint8_t* pass, int32_t n, int32_t* idx);

/* bf16 round-to-nearest-even of a double (8 significant bits). */
double orc_round_bf16(double x);

/* Single 3x3 convolution layer, stride 1, zero padding 1, cross-correlation (C6):
 * out[k][y][x] = b[k] + sum_{c,dy,dx} in[c][y+dy-1][x+dx-1] * w[k][c][dy][dx]. CHW fp64. b may be NULL. */
void orc_conv3x3(const double* in, int32_t C, int32_t H, int32_t W, const double* w, const double* b, int32_t K,
                 double* out);
/* 2x2 max-pool, stride 2, floor (C6). */
void orc_maxpool2(const double* in, int32_t C, int32_t H, int32_t W, double* out);

/* C5 + C6 ("SNM is a three-layer CNN (CONV, CONV, and FC)"; L167 50x50 input; Q9-Q11, Q15):
 * x[c][y][x] = (d50[y][x][c] - 128) / 128; conv1 (3->c1) + b1 -> ReLU -> maxpool2 -> [bf16] -> conv2 (c1->c2)
 * + b2 -> ReLU -> maxpool2 -> FC (F -> 1) + bfc. params = w1[c1][3][3][3], b1[c1], w2[c2][c1][3][3], b2[c2],
 * wfc[F], bfc[1]. bf16_emul = 1 rounds w1, w2, wfc and the pooled conv1 output to bf16 (the kernel's
 * operand precision); 0 is the plain fp64 network. Returns the logit. */
double orc_snm_forward(const uint8_t* d50, int32_t h, int32_t w, const float* params, int32_t c1, int32_t c2,
                       int32_t bf16_emul);
int64_t orc_snm_n_params(int32_t h, int32_t w, int32_t c1, int32_t c2);

/* C7 (Eq. (2)): t_pre = (c_high - c_low) * FilterDegree + c_low. */
double orc_tpre(double c_low, double c_high, double filter_degree);
/* logit-space threshold ln(t / (1 - t)); -inf at t = 0, +inf at t = 1. */
double orc_logit(double t);
/* C7 (PAPER.md L159 three classes; L165 "c >= t_pre into the T-YOLO queue"): c = sigmoid(logit);
 * pass iff c >= t_pre; cls = 0 if c < c_low, 2 if c > c_high, else 1. All compared in logit space. */
void orc_decide(double logit, double c_low, double c_high, double filter_degree, uint8_t* pass, uint8_t* cls);

/* ---------------------------------------------------------------------------------------------------------
 * f1: Tiny-YOLO-VOC (T-YOLO) stage + NumberofObjects (§3.2.3, §4.2.2; DESIGN.md
 * readings Q28-Q32).
 * "T-YOLO consists of 9 CONV layers and 6 POOL layers" on "416*416 pixel images" (L169), trained on VOC's 20
 * classes; "divides the input image into a 13*13 grid ... Each grid cell predicts 5 bounding boxes and confidence
 * scores ... If the confidence score exceeds the threshold (e.g., 0.2), one target object is considered to
 * appear" (L171). The layers are those of tiny-yolo-voc (L169's [44]):
 *   conv3x3 3->16, pool2/2, 16->32, pool2/2, 32->64, pool2/2, 64->128, pool2/2, 128->256, pool2/2, 256->512,
 *   pool2/1, 512->1024, 1024->1024 (each conv + bias, leaky ReLU 0.1; batch norm folded into the bias),
 *   conv1x1 1024->125 linear = 5 boxes x (tx, ty, tw, th, objectness, 20 class logits) per cell.
 * Params packed per layer: w[Cout][Cin][k][k] then b[Cout] (9 layers, 15,858,717 floats). */

/* Resize for filters whose feature size may exceed the frame (T-YOLO's 416 vs 360-row frames; Q28): cell i of a
 * dimension S split in D covers [floor(iS/D), max(floor((i+1)S/D), floor(iS/D) + 1)) -- the C1 box when S >= D,
 * one source pixel per cell otherwise; value = (s + n/2) / n. */
void orc_resize(const uint8_t* frame, int32_t W, int32_t H, int64_t pitch, int32_t Dw, int32_t Dh, uint8_t* out);

/* 1x1 convolution (C -> K), CHW fp64; b may be NULL. */
void orc_conv1x1(const double* in, int32_t C, int32_t H, int32_t W, const double* w, const double* b, int32_t K,
                 double* out);
/* leaky ReLU, slope 0.1 for x < 0 (darknet's "leaky") */
void orc_leaky(double* v, int64_t n);
/* 2x2 max-pool, stride 1, output H x W: out[y][x] = max over the in-bounds of (y..y+1, x..x+1) (darknet pads the
 * right/bottom border with -inf, Q30). */
void orc_maxpool2_s1(const double* in, int32_t C, int32_t H, int32_t W, double* out);

/* T-YOLO forward on a S x S x 3 u8 image (S = 416; any multiple of 32 for tests): x = v / 256 (Q29), the nine
 * layers above; bf16_emul = 1 rounds every weight and every layer's output activation to bf16 (the kernel's
 * operand precision). out = (S/32) x (S/32) x 125 doubles, HWC. Returns 0, or -1 if S is not a multiple of 32. */
int32_t orc_tyolo_forward(const uint8_t* img, int32_t S, const float* params, int32_t bf16_emul, double* out);
int64_t orc_tyolo_n_params(void);

/* L171 + L195 (NumberofObjects): score of box b of a cell = sigmoid(objectness) * softmax(class logits)[target];
 * a target object appears in the box iff score > thresh (strict, "exceeds"); returns the count over all cells and
 * boxes (Q31: no non-maximum suppression). A frame passes T-YOLO iff count >= NumberofObjects. */
int32_t orc_tyolo_count(const double* out, int32_t cells, int32_t target_class, double thresh);

#endif
