/*
 * cpubase/omp.c -- the all-cores OpenMP CPU BASELINE of SURVEY.md 8(d)
 * ("(2) The OpenMP baseline runs on all host cores ... a baseline, never a
 * reference").  It is timed by bench.py beside the single-thread oracle and
 * is checked against the oracle by tests/test_cpubase.py; it is NOT the
 * oracle (oracle/xro.c is) and it is not the product (the CUDA path is).
 * It shares no code with either.
 *
 * What it computes: the same reduction as xr_reduce (PAPER.md @4654-4854:
 * one associative operator over the reduced levels of the k/j/i nest,
 * @9947-10334; one result per kept iteration, @17176; the original value
 * merged after the reduction, @21828-21990), in the way a CPU OpenMP code
 * would:
 *   - the outermost non-unit level p is split into nthreads contiguous
 *     blocks (static schedule) -- the paper's gang "blocking" (@26322);
 *   - each thread runs the k -> j -> i loops of its block and accumulates IN
 *     THE DATA TYPE (fp32 in fp32, ints wrapping as unsigned) into private
 *     accumulators (p reduced) or straight into its own disjoint outputs
 *     (p kept);
 *   - private accumulators are combined in thread order 0..T-1, then the
 *     initial value is merged: out = init (+) R.
 * Operator semantics follow the readings C4 (identities), C6 (wrap), C7 (fp
 * max/min: NaN ignored, -0 < +0), C8 (&& || truth x != 0, result 0/1).
 * fp + and * reassociate relative to the oracle (C9/C10 tolerances apply).
 *
 * Build: gcc -O3 -fopenmp -ffp-contract=off -shared -fPIC cpubase/omp.c
 */
#include <math.h>
#include <omp.h>
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

enum { B_ADD, B_MUL, B_MAX, B_MIN, B_AND, B_OR, B_XOR, B_LAND, B_LOR };
enum { B_I32, B_I64, B_F32, B_F64 };
#define B_INIT_FROM_OUT 0x100u

/* -------------------------------------------------------------- operators */
static inline float f32_max(float a, float b) {
  return isnan(b) ? a : isnan(a) ? b : a == b ? (signbit(a) ? b : a) : (a > b ? a : b);
}
static inline float f32_min(float a, float b) {
  return isnan(b) ? a : isnan(a) ? b : a == b ? (signbit(a) ? a : b) : (a < b ? a : b);
}
static inline double f64_max(double a, double b) {
  return isnan(b) ? a : isnan(a) ? b : a == b ? (signbit(a) ? b : a) : (a > b ? a : b);
}
static inline double f64_min(double a, double b) {
  return isnan(b) ? a : isnan(a) ? b : a == b ? (signbit(a) ? a : b) : (a < b ? a : b);
}
static inline uint32_t i32_max(uint32_t a, uint32_t b) { return (int32_t)a > (int32_t)b ? a : b; }
static inline uint32_t i32_min(uint32_t a, uint32_t b) { return (int32_t)a < (int32_t)b ? a : b; }
static inline uint64_t i64_max(uint64_t a, uint64_t b) { return (int64_t)a > (int64_t)b ? a : b; }
static inline uint64_t i64_min(uint64_t a, uint64_t b) { return (int64_t)a < (int64_t)b ? a : b; }

/* One instantiation per dtype: T = element type, U = accumulator type
 * (unsigned for ints so + * wrap without UB). */
#define DEFINE_KERNEL(NAME, T, U, LOWEST, HIGHEST)                                  \
  static U NAME##_identity(int op) {                                                   \
    switch (op) {                                                                      \
      case B_MUL: case B_LAND: return (U)1;                                            \
      case B_MAX: return (U)(LOWEST);                                                  \
      case B_MIN: return (U)(HIGHEST);                                                 \
      case B_AND: return (U)~(uint64_t)0;                                              \
      default: return (U)0;                                                            \
    }                                                                                  \
  }                                                                                    \
  static inline U NAME##_comb(int op, U a, U b) {                                      \
    switch (op) {                                                                      \
      case B_ADD: return a + b;                                                        \
      case B_MUL: return a * b;                                                        \
      case B_MAX: return NAME##_max(a, b);                                             \
      case B_MIN: return NAME##_min(a, b);                                             \
      case B_LAND: return (U)(a != 0 && b != 0);                                       \
      case B_LOR: return (U)(a != 0 || b != 0);                                        \
    }                                                                                  \
    return NAME##_bits(op, a, b);                                                      \
  }                                                                                    \
  /* fold a contiguous run x[0..n) into acc (same output) */                           \
  static U NAME##_run(int op, U acc, const T* x, int64_t n) {                          \
    switch (op) {                                                                      \
      case B_ADD: { U s = 0; _Pragma("omp simd reduction(+:s)") for (int64_t i = 0; i < n; ++i) s += (U)x[i]; return acc + s; } \
      case B_MUL: { U s = 1; _Pragma("omp simd reduction(*:s)") for (int64_t i = 0; i < n; ++i) s *= (U)x[i]; return acc * s; } \
      case B_LAND: { int t = acc != 0; for (int64_t i = 0; i < n; ++i) t &= x[i] != 0; return (U)t; } \
      case B_LOR: { int t = acc != 0; for (int64_t i = 0; i < n; ++i) t |= x[i] != 0; return (U)t; } \
      default: for (int64_t i = 0; i < n; ++i) acc = NAME##_comb(op, acc, (U)x[i]); return acc; \
    }                                                                                  \
  }                                                                                    \
  /* fold x[0..n) elementwise into acc[0..n) (n distinct outputs) */                   \
  static void NAME##_vec(int op, U* acc, const T* x, int64_t n) {                      \
    switch (op) {                                                                      \
      case B_ADD: for (int64_t i = 0; i < n; ++i) acc[i] += (U)x[i]; return;           \
      case B_MUL: for (int64_t i = 0; i < n; ++i) acc[i] *= (U)x[i]; return;           \
      default: for (int64_t i = 0; i < n; ++i) acc[i] = NAME##_comb(op, acc[i], (U)x[i]); return; \
    }                                                                                  \
  }                                                                                    \
  static void NAME##_reduce(int op, const int64_t n[3], unsigned mask, const T* in,    \
                            T* out, int nth) {                                         \
    int64_t cnt = 1, red = 1;                                                          \
    for (int d = 0; d < 3; ++d) { if ((mask >> d) & 1u) red *= n[d]; else cnt *= n[d]; } \
    int p = 0;                                                                         \
    while (p < 2 && n[p] == 1) ++p; /* outermost non-unit level */                     \
    const int p_red = (mask >> p) & 1u;                                                \
    const int gk = !(mask & 1u), wk = !(mask & 2u), vk = !(mask & 4u);                 \
    const int64_t s1 = wk ? (vk ? n[2] : 1) : 0; /* output stride of j */              \
    const int64_t s0 = gk ? (wk ? n[1] : 1) * (vk ? n[2] : 1) : 0; /* of k */          \
    U* priv = (U*)malloc(sizeof(U) * (size_t)(p_red ? cnt * nth : cnt));               \
    const U e = NAME##_identity(op);                                                   \
    if (p_red) /* every slot, in case fewer threads than nth are granted */           \
      for (int64_t q = 0; q < cnt * nth; ++q) priv[q] = e;                             \
    _Pragma("omp parallel num_threads(nth)") {                                         \
      const int t = omp_get_thread_num(), T_ = omp_get_num_threads();                  \
      const int64_t lo = n[p] * t / T_, hi = n[p] * (t + 1) / T_;                      \
      U* acc = p_red ? priv + (size_t)t * cnt : priv;                                  \
      int64_t b[3] = {0, 0, 0}, E[3] = {n[0], n[1], n[2]};                             \
      b[p] = lo; E[p] = hi;                                                            \
      if (!p_red) { /* this thread owns the outputs of its block */                    \
        for (int64_t k = b[0]; k < E[0]; ++k)                                          \
          for (int64_t j = b[1]; j < E[1]; ++j) {                                      \
            int64_t o0 = k * s0 + j * s1;                                              \
            if (vk) for (int64_t i = b[2]; i < E[2]; ++i) acc[o0 + i] = e;             \
            else acc[o0] = e;                                                          \
          }                                                                            \
        /* outputs whose loops are reduced were just set more than once: fine */      \
      }                                                                                \
      for (int64_t k = b[0]; k < E[0]; ++k)                                            \
        for (int64_t j = b[1]; j < E[1]; ++j) {                                        \
          const T* x = in + (k * n[1] + j) * n[2] + b[2];                              \
          int64_t o0 = k * s0 + j * s1;                                                \
          if (vk) NAME##_vec(op, acc + o0 + b[2], x, E[2] - b[2]);                     \
          else acc[o0] = NAME##_run(op, acc[o0], x, E[2] - b[2]);                      \
        }                                                                              \
    }                                                                                  \
    if (p_red) /* combine the private partials in thread order */                      \
      for (int t = 1; t < nth; ++t)                                                    \
        for (int64_t o = 0; o < cnt; ++o) priv[o] = NAME##_comb(op, priv[o], priv[(size_t)t * cnt + o]); \
    (void)red;                                                                         \
    for (int64_t o = 0; o < cnt; ++o) {                                                \
      U init = (mask & B_INIT_FROM_OUT) ? (U)out[o] : e;                               \
      if ((mask & B_INIT_FROM_OUT) && (op == B_LAND || op == B_LOR)) init = (U)(out[o] != 0); \
      U r = NAME##_comb(op, init, priv[o]);                                            \
      if (op == B_LAND || op == B_LOR) r = (U)(r != 0);                                \
      out[o] = (T)r;                                                                   \
    }                                                                                  \
    free(priv);                                                                        \
  }

static inline uint32_t i32_bits(int op, uint32_t a, uint32_t b) {
  return op == B_AND ? (a & b) : op == B_OR ? (a | b) : (a ^ b);
}
static inline uint64_t i64_bits(int op, uint64_t a, uint64_t b) {
  return op == B_AND ? (a & b) : op == B_OR ? (a | b) : (a ^ b);
}
static inline float f32_bits(int op, float a, float b) { (void)op; (void)b; return a; }
static inline double f64_bits(int op, double a, double b) { (void)op; (void)b; return a; }

/* ints: for max/min the accumulator holds the signed value's bits */
DEFINE_KERNEL(i32, int32_t, uint32_t, INT32_MIN, INT32_MAX)
DEFINE_KERNEL(i64, int64_t, uint64_t, INT64_MIN, INT64_MAX)
DEFINE_KERNEL(f32, float, float, -INFINITY, INFINITY)
DEFINE_KERNEL(f64, double, double, -INFINITY, INFINITY)

/* Returns 0 on success, 1 invalid, 2 unsupported (& | ^ on fp, reading C3).
 * in / out are host arrays; out holds one element per kept iteration
 * (read first when B_INIT_FROM_OUT is set).  nthreads <= 0: all cores. */
int xrb_reduce(int op, int dtype, const int64_t dims[3], unsigned mask, const void* in, void* out,
               int nthreads) {
  if (op < B_ADD || op > B_LOR || dtype < B_I32 || dtype > B_F64 || !(mask & 7u)) return 1;
  if ((dtype == B_F32 || dtype == B_F64) && (op == B_AND || op == B_OR || op == B_XOR)) return 2;
  for (int d = 0; d < 3; ++d)
    if (dims[d] <= 0) return 1; /* the baseline times non-empty nests only */
  int nth = nthreads > 0 ? nthreads : omp_get_num_procs();
  /* drop extent-1 levels and merge adjacent levels of equal status (row-major
   * adjacent levels are one contiguous level), right-aligned in 3 slots */
  int64_t g[3];
  int gr[3], ng = 0;
  for (int d = 0; d < 3; ++d) {
    if (dims[d] == 1) continue;
    int r = (mask >> d) & 1u;
    if (ng && gr[ng - 1] == r) g[ng - 1] *= dims[d];
    else { g[ng] = dims[d]; gr[ng] = r; ++ng; }
  }
  int64_t n[3] = {1, 1, 1};
  unsigned m = mask & B_INIT_FROM_OUT;
  for (int q = 0; q < ng; ++q) {
    n[3 - ng + q] = g[q];
    if (gr[q]) m |= 1u << (3 - ng + q);
  }
  if (!(m & 7u)) m |= 1u; /* only extent-1 levels were reduced */
  switch (dtype) {
    case B_I32: i32_reduce(op, n, m, (const int32_t*)in, (int32_t*)out, nth); break;
    case B_I64: i64_reduce(op, n, m, (const int64_t*)in, (int64_t*)out, nth); break;
    case B_F32: f32_reduce(op, n, m, (const float*)in, (float*)out, nth); break;
    default: f64_reduce(op, n, m, (const double*)in, (double*)out, nth); break;
  }
  return 0;
}

int xrb_num_procs(void) { return omp_get_num_procs(); }
