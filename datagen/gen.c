/* datagen/gen.c -- seeded synthetic inputs for the cSTF hot path.
 *
 * This module holds NONE of the method's arithmetic (no MTTKRP, Gram, ADMM,
 * normalisation or fit).  It only draws numbers.  Both the FP64 oracle
 * (oracle/) and the CUDA path (paper_conf_icpp_sohksc24_b200/) consume its
 * output; neither side imports the other.
 *
 * Generator:
 *   counter-based SplitMix64: u(seed, stream, t) in [0,1) with 53 bits.
 *   Nonzero t, mode n:
 *     rank = t                               if t < I_n (coverage pass: every slice non-empty)
 *     rank = min(floor(I_n * u^gamma_n), I_n-1) otherwise (power-law skew, gamma in {1,2,3})
 *     label = (a_n * rank + b_n) mod I_n      (gcd(a_n, I_n) = 1: scatters the hot rows)
 *   value  = 1 + (53 - bitlength(x_v)), x_v the 53-bit draw  (count-like: 1/2 ones, 1/4 twos, ...)
 * Shapes come from PAPER.md Table 2 (L917-928); the paper gives no value or
 * index distribution, so the recipe is ours.
 */
#include <stdint.h>
#include <math.h>

static inline uint64_t mix64(uint64_t z) {
  z ^= z >> 30; z *= 0xBF58476D1CE4E5B9ULL;
  z ^= z >> 27; z *= 0x94D049BB133111EBULL;
  z ^= z >> 31; return z;
}
static inline uint64_t stream_key(uint64_t seed, uint64_t stream) {
  return mix64(seed * 0x9E3779B97F4A7C15ULL ^ mix64(stream + 0xD1B54A32D192ED03ULL));
}
/* 64 random bits for counter t of (seed, stream). */
static inline uint64_t draw(uint64_t key, uint64_t t) {
  return mix64(key + (t + 1) * 0x9E3779B97F4A7C15ULL);
}
static inline double unit53(uint64_t bits) { return (double)(bits >> 11) * 0x1.0p-53; }

static int64_t gcd64(int64_t a, int64_t b) { while (b) { int64_t t = a % b; a = b; b = t; } return a; }

/* Multiplier/offset of the label scatter for a mode of length I. */
void datagen_scatter_params(int64_t I, int64_t* a, int64_t* b) {
  int64_t x = (int64_t)(0.6180339887498949 * (double)I) | 1;
  if (x < 1) x = 1;
  while (I > 1 && gcd64(x, I) != 1) x += 2;
  *a = (I > 1) ? (x % I) : 0;
  *b = (int64_t)(0.3141592653589793 * (double)I);
  if (I > 0) *b %= I;
}

void datagen_uniform(uint64_t seed, uint64_t stream, int64_t count, double* out) {
  uint64_t key = stream_key(seed, stream);
#pragma omp parallel for schedule(static)
  for (int64_t t = 0; t < count; t++) out[t] = unit53(draw(key, (uint64_t)t));
}

/* Fill one mode's indices for nonzeros [0, nnz). */
void datagen_mode_indices(uint64_t seed, int mode, int64_t I, int gamma, int64_t nnz, int32_t* out) {
  uint64_t key = stream_key(seed, (uint64_t)mode);
  int64_t a, b; datagen_scatter_params(I, &a, &b);
#pragma omp parallel for schedule(static)
  for (int64_t t = 0; t < nnz; t++) {
    int64_t rank;
    if (t < I) rank = t;
    else {
      double u = unit53(draw(key, (uint64_t)t));
      double p = u;
      for (int g = 1; g < gamma; g++) p = p * u;
      rank = (int64_t)floor((double)I * p);
      if (rank > I - 1) rank = I - 1;
    }
    out[t] = (int32_t)((a * rank + b) % I);
  }
}

void datagen_values(uint64_t seed, int64_t nnz, double* out) {
  uint64_t key = stream_key(seed, 100);
#pragma omp parallel for schedule(static)
  for (int64_t t = 0; t < nnz; t++) {
    uint64_t x = draw(key, (uint64_t)t) >> 11;  /* 53 bits */
    int bl = 0; while (x) { bl++; x >>= 1; }
    out[t] = (double)(1 + (53 - bl));
  }
}
