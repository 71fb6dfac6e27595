/*
 * datagen/gen.c -- seeded, counter-based synthetic input generator.
 *
 * This module is shared by BOTH sides of the parity check (the oracle under
 * oracle/ and the CUDA path under paper_conf_ppopp_xutycc14_b200/).  It holds
 * none of the method's arithmetic: it only turns (seed, global index) into
 * input values, so that a shard of an array generated at global indices
 * [start, start+n) is byte-identical to the same slice of the whole array
 * (SURVEY.md 8(d) "Generator"; 8(e) "each rank generates its shard").
 *
 * h(idx) = splitmix64(seed + idx * 0x9E3779B97F4A7C15)
 * Distributions:
 *   U_int[a,b]  = a + h mod (b-a+1)
 *   U_f32[a,b)  = a + (b-a) * ((h >> 40) * 2^-24)     (24-bit grid)
 *   U_f64[a,b)  = a + (b-a) * ((h >> 11) * 2^-53)     (53-bit grid)
 *   affine permutation of 0..n-1: (A*idx + B) mod n, gcd(A, n) = 1
 *
 * Build: gcc -O2 -fopenmp -shared -fPIC datagen/gen.c -o datagen/libxrgen.so
 */
#include <stdint.h>
#include <string.h>

#define XG_GOLDEN 0x9E3779B97F4A7C15ULL

static inline uint64_t xg_mix(uint64_t z) {
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
  return z ^ (z >> 31);
}

uint64_t xg_splitmix64(uint64_t x) { return xg_mix(x + XG_GOLDEN); }

static inline uint64_t xg_h(uint64_t seed, uint64_t idx) {
  return xg_mix(seed + idx * XG_GOLDEN);
}

uint64_t xg_hash(uint64_t seed, uint64_t idx) { return xg_h(seed, idx); }

void xg_hashes(uint64_t seed, int64_t start, int64_t n, uint64_t* out) {
#pragma omp parallel for schedule(static)
  for (int64_t t = 0; t < n; ++t) out[t] = xg_h(seed, (uint64_t)(start + t));
}

void xg_uniform_i32(uint64_t seed, int64_t start, int64_t n, int64_t a, int64_t b,
                    int32_t* out) {
  uint64_t span = (uint64_t)(b - a) + 1u;
#pragma omp parallel for schedule(static)
  for (int64_t t = 0; t < n; ++t)
    out[t] = (int32_t)(a + (int64_t)(xg_h(seed, (uint64_t)(start + t)) % span));
}

void xg_uniform_i64(uint64_t seed, int64_t start, int64_t n, int64_t a, int64_t b,
                    int64_t* out) {
  uint64_t span = (uint64_t)b - (uint64_t)a + 1u; /* 0 means the full 2^64 range */
#pragma omp parallel for schedule(static)
  for (int64_t t = 0; t < n; ++t) {
    uint64_t h = xg_h(seed, (uint64_t)(start + t));
    uint64_t r = span ? h % span : h;
    out[t] = (int64_t)((uint64_t)a + r);
  }
}

void xg_uniform_f32(uint64_t seed, int64_t start, int64_t n, double a, double b,
                    float* out) {
  const double scale = 1.0 / 16777216.0; /* 2^-24 */
#pragma omp parallel for schedule(static)
  for (int64_t t = 0; t < n; ++t) {
    uint64_t h = xg_h(seed, (uint64_t)(start + t));
    out[t] = (float)(a + (b - a) * ((double)(h >> 40) * scale));
  }
}

void xg_uniform_f64(uint64_t seed, int64_t start, int64_t n, double a, double b,
                    double* out) {
  const double scale = 1.0 / 9007199254740992.0; /* 2^-53 */
#pragma omp parallel for schedule(static)
  for (int64_t t = 0; t < n; ++t) {
    uint64_t h = xg_h(seed, (uint64_t)(start + t));
    out[t] = a + (b - a) * ((double)(h >> 11) * scale);
  }
}

/* values[t] = (A*(start+t) + B) mod m  -- a bijection of 0..m-1 when gcd(A,m)=1 */
void xg_affine_i64(int64_t start, int64_t n, uint64_t A, uint64_t B, uint64_t m,
                   int64_t* out) {
#pragma omp parallel for schedule(static)
  for (int64_t t = 0; t < n; ++t) {
    unsigned __int128 v = (unsigned __int128)A * (uint64_t)(start + t) + B;
    out[t] = (int64_t)(uint64_t)(v % m);
  }
}

void xg_affine_i32(int64_t start, int64_t n, uint64_t A, uint64_t B, uint64_t m,
                   int32_t* out) {
#pragma omp parallel for schedule(static)
  for (int64_t t = 0; t < n; ++t) {
    unsigned __int128 v = (unsigned __int128)A * (uint64_t)(start + t) + B;
    out[t] = (int32_t)(uint32_t)(uint64_t)(v % m);
  }
}

/* values[t] = (start + t) mod 2^w, stored in the target width (linear index). */
void xg_linear_i32(int64_t start, int64_t n, int32_t* out) {
#pragma omp parallel for schedule(static)
  for (int64_t t = 0; t < n; ++t) out[t] = (int32_t)(uint32_t)(uint64_t)(start + t);
}

void xg_linear_i64(int64_t start, int64_t n, int64_t* out) {
#pragma omp parallel for schedule(static)
  for (int64_t t = 0; t < n; ++t) out[t] = start + t;
}

/* sel[t] = 1 iff h(seed, start+t) mod den < num : a Bernoulli(num/den) mask used
 * to plant special values at hash-chosen global indices (rate scaled to the
 * segment length by the caller, SURVEY.md 8(d) cfg5 recipe). */
void xg_select(uint64_t seed, int64_t start, int64_t n, uint64_t num, uint64_t den,
               uint8_t* sel) {
#pragma omp parallel for schedule(static)
  for (int64_t t = 0; t < n; ++t)
    sel[t] = (uint8_t)((xg_h(seed, (uint64_t)(start + t)) % den) < num);
}
