/*
 * oracle/xro.h -- TEST INFRASTRUCTURE ONLY.
 *
 * Plain, slow, sequential CPU oracle for the hot path of Xu et al.,
 * "Reduction Operations in Parallel Loops for GPGPUs" (PMAM'14), PAPER.md.
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline /
 * --impl reference legs may load it.  It shares NO code with the CUDA path
 * (paper_conf_ppopp_xutycc14_b200/): enums and status codes are deliberately
 * re-declared here and cross-checked by a test.
 *
 * Definition followed (SURVEY.md 8(c) "Plain definition"):
 *   out[o] = init[o] (+) OP_{r in prod_{d in R}[0,n_d)} in[compose(o, r)]
 * where R = reduced levels (mask bits), o ranges row-major over the kept
 * levels in (k, j, i) order, init = identity or the prior out[o]
 * (XRO_INIT_FROM_OUT, the paper's "original value", PAPER.md @21488-21990,
 * "the initial value is processed after the vector reduction algorithm is
 * done ... summed for + or multiplied for *").
 * Any evaluation order is licensed by associativity + commutativity
 * (PAPER.md @15024-15239, section 3); the oracle uses the paper's nest order
 * k -> j -> i (Fig 3/4, @13404, @16410) and the paper's own check, "perform
 * reduction ... then on the CPU side ... compare" (@37147-37270).
 *
 * Parity pins: see tests/test_oracle_pins.py (P1-P16 of SURVEY.md 8(c)).
 * The heat function follows Fig 13(a) (@43561-44280) under reading C14.
 */
#ifndef XRO_H
#define XRO_H
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* op codes: + * max min & | ^ && ||   (reading C1) */
enum { XRO_ADD = 0, XRO_MUL = 1, XRO_MAX = 2, XRO_MIN = 3, XRO_BAND = 4,
       XRO_BOR = 5, XRO_BXOR = 6, XRO_LAND = 7, XRO_LOR = 8 };
/* operand types: int / float / double of Table 2, plus int64 (reading C2) */
enum { XRO_I32 = 0, XRO_I64 = 1, XRO_F32 = 2, XRO_F64 = 3 };
/* level bits: gang = dims[0] (k, outermost), worker = dims[1] (j),
 * vector = dims[2] (i, contiguous)   (PAPER.md @10459-11313, Fig 3) */
#define XRO_GANG 0x1u
#define XRO_WORKER 0x2u
#define XRO_VECTOR 0x4u
#define XRO_INIT_FROM_OUT 0x100u
enum { XRO_OK = 0, XRO_ERR_INVALID = 1, XRO_ERR_UNSUPPORTED = 2 };

/* Number of outputs: product of the kept extents (1 if every level reduced). */
int xro_out_count(const int64_t dims[3], unsigned mask, int64_t* count);

/* Reduce in[k][j][i] (row-major, dims = {n0, n1, n2}) over the levels in mask.
 * out: xro_out_count elements of dtype (read first if XRO_INIT_FROM_OUT).
 * abs_sum (nullable): per output |init| + sum |x|, for the fp tolerance (C9). */
int xro_reduce(int op, int dtype, const int64_t dims[3], unsigned mask,
               const void* in, void* out, double* abs_sum);

/* Transform-reduce, two inputs x, y of the same nest:
 *  XRO_XF_DISK: Monte Carlo pi, Fig 13(c) (PAPER.md @43561-44280, 4. @42177-
 *    47503): out[o] (int64) = init + #{ r : x*x + y*y < 1 }, the products and
 *    the sum rounded in dtype (fp32 / fp64), no FMA (the paper disables FMA,
 *    @35389) -- the predicate is decided in the same precision on both sides.
 *  XRO_XF_DOT: inner product, Fig 13(b) (@41386-42177): out[o] (dtype) =
 *    init + sum_r x*y, ints wrapping, fp in wide precision (C9 bound).
 * abs_sum (nullable, DOT only): |init| + sum |x*y| per output. */
enum { XRO_XF_DISK = 1, XRO_XF_DOT = 2 };
int xro_transform_reduce(int xform, int dtype, const int64_t dims[3], unsigned mask,
                         const void* x, const void* y, void* out, double* abs_sum);

/* Heat equation (config 4, reading C14): T[j][i], nj x ni, row-major fp64. */
int xro_heat_init(int64_t nj, int64_t ni, double* T);
/* iters Jacobi sweeps starting from T1 (T2 must carry the same boundary);
 * residuals[it] = max over all points of |T_new - T_old| of sweep it.
 * The newest field is in T1 when iters is even, in T2 when odd. */
int xro_heat(int64_t nj, int64_t ni, int64_t iters, double* T1, double* T2,
             double* residuals);

#ifdef __cplusplus
}
#endif
#endif
