/*
 * include/xreduce.h -- C ABI of xreduce, the B200-native (sm_100a) hot path of
 * Xu et al., "Reduction Operations in Parallel Loops for GPGPUs" (PMAM'14).
 *
 * Citations are PAPER.md:1 character offsets (@N; the extracted paper is one
 * line) with the section they fall in.  See DESIGN.md for the readings C1-C23
 * adopted where the paper is silent or garbled.
 *
 * The problem (PAPER.md @4654-4854, section 1; again @13077-13277, section 3):
 * "a binary associative operator to operate an input array and generate a
 * single output value", placed on any of the three loop levels of a nest
 * (gang = outer k, worker = middle j, vector = inner i; @9947-10334, 2.2) or
 * on several of them (RMP, @26751-27253, 3.2).  Levels that are not reduced
 * "execute in parallel" (@44766, Table 2 caption) and yield one result per
 * iteration (Fig 4: temp[k][j][0] = i_sum, @17176).  The variable's original
 * value is combined after the reduction (@21488-21990, 3.1.1).
 *
 * Conventions (every entry point):
 *  - Return an xr_status; 0 = success.  No C++ exception crosses the ABI.
 *  - Argument validation runs BEFORE any CUDA call, so invalid calls return
 *    XR_ERR_INVALID / XR_ERR_UNSUPPORTED on machines without a GPU.
 *  - Device calls are asynchronous on `stream` (a cudaStream_t; NULL = legacy
 *    default stream); results are valid after the stream synchronises.  No
 *    host synchronisation happens inside xr_reduce except when the library's
 *    workspace must grow (first calls only; see xr_reserve).
 *  - Thread-safe across host threads.  Concurrent calls on DIFFERENT streams
 *    use different workspaces.
 */
#ifndef XREDUCE_H
#define XREDUCE_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* Compatible with cudaStream_t (both are `struct CUstream_st *`). */
typedef struct CUstream_st* xr_stream_t;

/* Opaque NCCL communicator of the multi-GPU entry points (xr_comm_init). */
typedef struct xr_comm_s* xr_comm_t;

/* Operators (reading C1: the OpenACC C set; the paper evaluates + and *
 * (@37852-37985) and max (@37985, Fig 13a) and claims "all reduction
 * operator types" (@6300-6414)). */
typedef enum {
  XR_OP_ADD = 0,  /* +   identity 0 (+0.0 for fp)                           */
  XR_OP_MUL = 1,  /* *   identity 1                                          */
  XR_OP_MAX = 2,  /* max identity lowest (INT_MIN / -inf); fp: NaN operands
                     ignored, -0 < +0 (reading C7)                           */
  XR_OP_MIN = 3,  /* min identity highest (INT_MAX / +inf); same fp rule     */
  XR_OP_BAND = 4, /* &   identity ~0        (integers only, reading C3)      */
  XR_OP_BOR = 5,  /* |   identity 0         (integers only)                  */
  XR_OP_BXOR = 6, /* ^   identity 0         (integers only)                  */
  XR_OP_LAND = 7, /* &&  identity 1; truth = (x != 0); result 0/1 in dtype (C8) */
  XR_OP_LOR = 8   /* ||  identity 0; result 0/1 in dtype                     */
} xr_op;

/* Operand types: Table 2's int / float / double (@45106-45160) plus int64
 * (reading C2).  The output has the input's type.  Integer + and * wrap
 * modulo 2^32 / 2^64 (reading C6). */
typedef enum { XR_INT32 = 0, XR_INT64 = 1, XR_FP32 = 2, XR_FP64 = 3 } xr_dtype;

/* Level bits of `level_mask`.  nest_dims = {n0, n1, n2} describes the
 * row-major array in[k][j][i] with k < n0 (gang, outermost), j < n1 (worker),
 * i < n2 (vector, contiguous) -- the paper's mapping "k loop ... across all
 * gangs, j ... across all workers ..., i ... across all vector threads"
 * (@10531-11313, Fig 2/3). */
#define XR_GANG 0x1u
#define XR_WORKER 0x2u
#define XR_VECTOR 0x4u
/* out[] holds per-output initial values (the paper's "original value",
 * @21488-21990); otherwise the initial value is the identity. */
#define XR_INIT_FROM_OUT 0x100u

typedef enum {
  XR_OK = 0,
  XR_ERR_INVALID = 1,     /* bad op/dtype code, mask, dims, pointer, overlap  */
  XR_ERR_UNSUPPORTED = 2, /* & | ^ on fp32/fp64 (reading C3)                  */
  XR_ERR_CUDA = 3,        /* a CUDA runtime error (launch, allocation, copy)  */
  XR_ERR_NCCL = 4,        /* an NCCL error (sharded calls)                    */
  XR_ERR_NOMEM = 5        /* workspace allocation failed                      */
} xr_status;

/* ---------------------------------------------------------------- core ---- */

/* xr_reduce -- out[o] = init[o] (+) OP over the reduced levels of in.
 *
 *   op, dtype   : xr_op, xr_dtype.  30 legal pairs: + * max min && || on all
 *                 four types, & | ^ on int32/int64 (else XR_ERR_UNSUPPORTED).
 *   nest_dims   : host pointer to 3 extents n0, n1, n2 >= 0 whose product
 *                 fits in int64 (else XR_ERR_INVALID).
 *   level_mask  : OR of XR_GANG / XR_WORKER / XR_VECTOR (at least one),
 *                 optionally | XR_INIT_FROM_OUT; other bits -> XR_ERR_INVALID.
 *                 Every combination is defined, including gang+vector without
 *                 worker (reading C13; the paper says it "cannot span across
 *                 gang & vector without going through the worker", @29561).
 *   in          : DEVICE pointer, n0*n1*n2 elements, dtype-aligned (4 or 8 B;
 *                 16 B alignment is NOT required).  Caller-owned, read only.
 *   out         : DEVICE pointer, xr_out_count elements, compact row-major over
 *                 the kept levels in (k, j, i) order (reading C11).  Must not
 *                 overlap in (XR_ERR_INVALID).  Read first when
 *                 XR_INIT_FROM_OUT is set, then overwritten.
 *   stream      : launch stream.
 * A kept extent of 0 gives an empty output (no-op).  A reduced extent of 0
 * gives out = init (reading C17).  Null pointers with non-empty work ->
 * XR_ERR_INVALID.  One kernel launch per call (single pass: per-CTA partials
 * combined by the last CTA to finish, no second launch). */
int xr_reduce(int op, int dtype, const int64_t nest_dims[3], unsigned level_mask,
              const void* in, void* out, xr_stream_t stream);

/* Number of outputs: the product of the kept extents (1 if all reduced). */
int xr_out_count(const int64_t nest_dims[3], unsigned level_mask, int64_t* count);

/* Static string for a status code (never NULL). */
const char* xr_strerror(int status);

/* Same as xr_reduce but with HOST buffers (pinned or pageable; pinned gives
 * the full PCIe rate).  The input is copied in bounded chunks (at most 32 MiB
 * each, XR_HOST_CHUNK_BYTES overrides) through TWO library-owned device
 * staging buffers on an internal copy stream, so the H2D copy of chunk c+1
 * overlaps the reduction of chunk c on `stream`.  Chunks run along the
 * outermost level whose single index fits in a chunk (earlier levels are
 * iterated one index at a time); a chunk's outputs are one contiguous block of
 * out.  When
 * the chunk level or a level before it is REDUCED, several chunks share an
 * output block: the first writes it (merging the caller's init), the later
 * ones combine into it (their init is the block's current value) -- the gang
 * tier across chunks, exact for integer / bitwise / logical / min / max and
 * within C9 / C10 for fp + and *.  Staging is owned per (device, stream): the
 * input buffers are 2 x min(chunk, input bytes), plus a device copy of the
 * output (xr_out_count elements).  Synchronous: returns after out (host) is
 * written; `stream` orders the work (NULL = legacy stream); concurrent calls
 * on different streams use different staging.  Errors as xr_reduce. */
int xr_reduce_host(int op, int dtype, const int64_t nest_dims[3], unsigned level_mask,
                   const void* in_host, void* out_host, xr_stream_t stream);

/* Host-only (no CUDA): the chunks xr_reduce_host would use with a chunk cap
 * of cap_bytes.  Writes up to max_chunks rows of 6 int64 to out6: chunk dims
 * n0, n1, n2, input offset (elements), output offset (elements), and 1 if the
 * chunk is the first to write its output block.  *nchunks = total count. */
int xr_host_chunks(const int64_t nest_dims[3], unsigned level_mask, int dtype, int64_t cap_bytes,
                   int64_t max_chunks, int64_t* out6, int64_t* nchunks);

/* Transform-reduce (the loop body before the reduction), two
 * inputs of the same nest (DEVICE, dtype-aligned, caller-owned):
 *   XR_XF_DISK  Monte Carlo pi, Fig 13(c) (@43561-44280, section 4
 *               @42177-47503): out[o] = init + #{ x*x + y*y < 1 } as int64,
 *               every operation rounded in dtype (fp32/fp64 only; other dtypes
 *               XR_ERR_UNSUPPORTED), no FMA (@35389).  out is int64.
 *   XR_XF_DOT   inner product, Fig 13(b) (@41386-42177): out[o] = init +
 *               sum x*y in dtype (ints wrap, C6; fp within the C9 bound).
 * level_mask as xr_reduce; every canonical shape (R, KR, RK, KRK, RKR, K) is
 * supported.  Column shapes (the reduced levels all outside a kept contiguous
 * level) read 16-B vectors of both inputs when both are 16-B aligned and the
 * kept row is a multiple of 16 B, else scalars.  One launch, single pass. */
typedef enum { XR_XF_DISK = 1, XR_XF_DOT = 2 } xr_xform;
int xr_transform_reduce(int xform, int dtype, const int64_t nest_dims[3], unsigned level_mask,
                        const void* x, const void* y, void* out, xr_stream_t stream);

/* Several reduction variables with mixed dtypes in ONE pass (
 * PAPER.md 3.3 @31605-32570: one reduction clause with e.g. an int and a float
 * variable sharing one shared-memory pool sized for the largest type).  Each
 * variable has its own op, dtype, input (DEVICE, n0*n1*n2 elements) and output
 * (DEVICE, xr_out_count elements); all share nest_dims and level_mask (with
 * XR_INIT_FROM_OUT applying to every output).  1 <= nvars <= 8.  Semantics per
 * variable exactly as xr_reduce; no output may overlap an input or another
 * output.  Every canonical shape (R, KR, RK, KRK, RKR, K) and empty extents
 * are supported.  One launch (none if every output is empty).
 * Errors (nothing is launched): XR_ERR_INVALID for nvars outside [1, 8], a
 * bad op / dtype / mask, a null or misaligned pointer with non-empty work, or
 * overlapping buffers; XR_ERR_UNSUPPORTED for & | ^ on fp; XR_ERR_CUDA if the
 * launch fails. */
typedef struct {
  int op;          /* xr_op   */
  int dtype;       /* xr_dtype */
  const void* in;
  void* out;
} xr_var;
int xr_reduce_multi(int nvars, const xr_var* vars, const int64_t nest_dims[3], unsigned level_mask,
                    xr_stream_t stream);

/* Different variables reduced at DIFFERENT levels of one nest, in one launch
 * (PAPER.md 3.2 @27198-27253: "reduction can also occur on different
 * variables within different levels of parallelism", e.g. i_sum at the vector
 * level and j_sum at the worker level of the same nest).
 * As xr_reduce_multi, but each variable carries its own level_mask (any legal
 * xr_reduce mask, XR_INIT_FROM_OUT per variable) and its output holds
 * xr_out_count(nest_dims, level_mask) elements of its dtype.  Each variable's
 * result is exactly xr_reduce(op, dtype, nest_dims, level_mask, in, out).
 * Variables may share an input (e.g. row sums and the total of one array);
 * outputs may not overlap any input or another output.  Errors as
 * xr_reduce_multi.  One launch. */
typedef struct {
  int op;               /* xr_op    */
  int dtype;            /* xr_dtype */
  unsigned level_mask;  /* XR_GANG | XR_WORKER | XR_VECTOR [| XR_INIT_FROM_OUT] */
  const void* in;
  void* out;
} xr_var_at;
int xr_reduce_multi_at(int nvars, const xr_var_at* vars, const int64_t nest_dims[3], xr_stream_t stream);

/* The paper's own code-generation scheme, an in-house A/B
 * baseline on the same GPU: Kepler-style launch of num_gangs blocks of
 * (vector_length x num_workers) threads (<= 0 selects the paper's 192 x (128 x
 * 8), @35893-36486), Fig 3 loops, shared-memory interleaved log-step trees
 * (Figs 6c, 7, 8c) and, when the gang level reduces, a global partial buffer
 * plus a SECOND kernel launch (Fig 5c, @24887-25280; RMP @30925-31587).
 * Masks XR_GANG, XR_WORKER, XR_VECTOR (the testsuite's single-level
 * positions) and the three RMP scenarios of 3.2.1 (@28973-29561): gang &
 * worker (global buffer of gangs x workers per output + second launch),
 * worker & vector (shared-memory buffer of workers x vectors), gang & worker &
 * vector (global buffer of every thread + second launch); gang & vector, which
 * the paper says "cannot span ... without going through the worker", returns
 * XR_ERR_UNSUPPORTED.  Ops + * max; dtypes int32, fp32, fp64 (Table 2).  Other
 * combinations: XR_ERR_UNSUPPORTED.  Same output layout and init semantics as
 * xr_reduce.  Two launches when gang reduces. */
int xr_reduce_paper(int op, int dtype, const int64_t nest_dims[3], unsigned level_mask, const void* in,
                    void* out, int num_gangs, int num_workers, int vector_length, xr_stream_t stream);

/* ------------------------------------------------------------ planning ---- */

/* Canonical shapes after dropping extent-1 levels and merging adjacent levels
 * of the same status.  R = reduced run, K = kept run. */
typedef enum {
  XR_SHAPE_NONE = 0,  /* empty output: nothing to do                        */
  XR_SHAPE_FILL = 1,  /* a reduced extent is 0: out = init                  */
  XR_SHAPE_IDENT = 2, /* "K": every reduced extent is 1: out = init (+) in  */
  XR_SHAPE_R = 3,     /* whole-nest scalar                                   */
  XR_SHAPE_KR = 4,    /* keep outer, reduce contiguous inner (rows)          */
  XR_SHAPE_RK = 5,    /* reduce outer, keep contiguous inner (columns)       */
  XR_SHAPE_KRK = 6,   /* batched columns                                     */
  XR_SHAPE_RKR = 7    /* keep the middle, reduce outer and inner             */
} xr_shape;

typedef struct {
  int shape;            /* xr_shape                                          */
  int kernel;           /* 0 none, 1 fill, 2 ident, 3 seg, 4 col, 5 stream,
                           6 coltma (TMA tensor-map column kernel),
                           7 rows (bulk-streamed short contiguous rows),
                           8 colflat (narrow-row column reduction),
                           9 rkr (bulk-streamed j-blocks of short rows, k loop),
                           10 colsmall (warp per 32 B of columns, small inputs),
                           11 rcluster (one 16-CTA cluster, DSMEM gang tier),
                           12 shortrow (thread per chunk of short rows),
                           13 thincol (thread per column group, few rows) */
  int64_t cdims[3];     /* canonical extents (shape-dependent, rest 0)       */
  int64_t out_count;
  int group;            /* seg: lanes per group (8, 32 or the CTA size)      */
  int vec;              /* elements per 16-byte load (col: 1 if unaligned)    */
  int64_t splits;       /* partial units per output (1 = no gang-tier combine) */
  int64_t units;        /* total work units                                  */
  int64_t grid;         /* CTAs launched                                     */
  int block;            /* threads per CTA                                   */
  int64_t ws_bytes;     /* workspace bytes (partials)                        */
  int64_t tickets;      /* last-CTA tickets                                  */
} xr_plan_info;

/* Host-only: the plan xr_reduce would use on a device with `num_sms` SMs.
 * `in_addr` is the input address (only its alignment matters).  No CUDA. */
int xr_plan_describe(int op, int dtype, const int64_t nest_dims[3], unsigned level_mask,
                     uint64_t in_addr, int num_sms, xr_plan_info* info);

/* Pre-grow the workspace of (current device, stream) for the given call so
 * that later calls never allocate (e.g. before CUDA-graph capture). */
int xr_reserve(int op, int dtype, const int64_t nest_dims[3], unsigned level_mask,
               xr_stream_t stream);

/* Release every workspace and staging buffer (synchronises the device). */
int xr_shutdown(void);

/* Number of kernels this library has launched in this process. */
int64_t xr_launch_count(void);

/* Profiling only: while buf (DEVICE, 2 + 2*cap_records uint64 words) is set,
 * the stream kernel appends per-CTA timeline records -- word 0 = records
 * written (the caller zeroes it), word 1 = cap_records (the caller writes
 * it), then per record {cta << 40 | event << 32 | unit, %globaltimer ns} with
 * events 0 CTA start, 1 unit claimed, 2 unit folded, 3 consumers done, 4 last
 * CTA fold begins, 5 output written.  buf = NULL switches it off. */
int xr_debug_timeline(void* buf, int64_t cap_records);

/* --------------------------------------------------------- heat (cfg 4) ---- */

/* One fused Jacobi sweep + max-residual reduction of the 2-D heat equation
 * (Fig 13(a) @43561-44280, section 4 @39322-41386; reading C14):
 *   T2[j][i] = 0.25*((T1[j-1][i] + T1[j+1][i]) + (T1[j][i-1] + T1[j][i+1]))
 * for 1 <= j < nj-1, 1 <= i < ni-1 (no FMA contraction), and
 *   *residual = max(0, max |T2 - T1|)   (gang+worker+vector max, one launch).
 * T1, T2: DEVICE nj x ni row-major fp64; T2's boundary must already hold the
 * boundary values (it is never written).  residual: DEVICE pointer to 1 fp64. */
int xr_heat_step(int64_t nj, int64_t ni, const double* T1, double* T2, double* residual,
                 xr_stream_t stream);

/* iters sweeps, swapping T1/T2; residuals[it] (DEVICE, iters fp64).  The
 * newest field is in T1 when iters is even, in T2 when odd. */
int xr_heat_run(int64_t nj, int64_t ni, int64_t iters, double* T1, double* T2,
                double* residuals, xr_stream_t stream);

/* Gang-row sharded heat (config 4 on several GPUs).  Rank r of
 * nranks owns global rows [r*n_local, (r+1)*n_local) of the
 * (nranks*n_local) x ni grid, stored in a DEVICE buffer of (n_local+2) x ni
 * fp64: local row 0 = global row r*n_local-1 and local row n_local+1 = global
 * row (r+1)*n_local are halos (unused at the global boundary).  Both buffers
 * must start with the initial field AND the neighbours' halo rows.  One step =
 * the fused sweep of the owned interior rows, then the halo rows of T2 are
 * exchanged with grouped ncclSend/ncclRecv and the residual is combined with
 * ncclAllReduce(max) of one fp64 into *residual (DEVICE) on every rank (also
 * at 1 rank).  The results are bit-identical to xr_heat_step on the whole
 * grid.  With XR_FORCE_COLL set and 1 rank (tests), the rank exchanges its
 * halos with itself: halo row 0 <- owned row 1, halo row n_local+1 <- owned
 * row n_local (both halos are unused at the global boundary). */
int xr_heat_step_sharded(int64_t n_local, int64_t ni, const double* T1, double* T2,
                         double* residual, xr_comm_t comm, xr_stream_t stream);
/* iters steps swapping T1/T2 (residuals: DEVICE, iters fp64), overlapped:
 * each sweep computes its two boundary rows first, the halo exchange of those
 * rows runs on the communicator's internal stream while the interior rows
 * sweep, and the residual allreduce of sweep k is issued after the halos of
 * sweep k+1 (one sweep late, hidden behind the next interior sweep).  When the
 * work enqueued on `stream` completes, every residuals[k] is final and
 * bit-identical to the serial xr_heat_step_sharded sequence (max is exact);
 * only a host that polled residuals[k] mid-run would see it one sweep late. */
int xr_heat_run_sharded(int64_t n_local, int64_t ni, int64_t iters, double* T1, double* T2,
                        double* residuals, xr_comm_t comm, xr_stream_t stream);
/* Single-device simulation of the same protocol over nranks slabs (halo
 * exchange by device copies, residual by the fixed-order max combine). */
int xr_heat_run_sharded_sim(int64_t n_local, int64_t ni, int64_t iters, int nranks,
                            double* const* T1s, double* const* T2s, double* residuals,
                            xr_stream_t stream);

/* ------------------------------------------------- multi-GPU (gang shards) */

/* Sharding along the gang level: rank r owns the contiguous
 * gang slice [r*n0_local, (r+1)*n0_local); every rank passes the same
 * local_dims.  After the call, out on EVERY rank holds the GLOBAL result:
 *   G in mask : xr_out_count(local_dims) elements (partials combined);
 *   G not in  : nranks * xr_out_count(local_dims) elements, rank-major
 *               (= global row-major, because gang is outermost).
 * XR_INIT_FROM_OUT with G in mask merges rank 0's init exactly once; with G
 * not in mask each rank merges the init of its own segment. */
typedef enum {
  XR_COLL_NONE = 0,
  XR_COLL_ALLREDUCE = 1,        /* ncclSum/Prod/Max/Min (&& -> Min, || -> Max on 0/1) */
  XR_COLL_ALLGATHER_COMBINE = 2,/* & | ^ : gather partials, fixed rank-order combine  */
  XR_COLL_ALLGATHER = 3         /* gang kept: gather disjoint output segments          */
} xr_collective;

typedef struct {
  int collective;        /* xr_collective                                    */
  int nccl_op;           /* ncclRedOp_t for XR_COLL_ALLREDUCE, else -1        */
  int merge_init;        /* 1 if this rank merges the caller's init locally   */
  int local_init_from_out; /* 1 if the local reduction reads out as init      */
  int64_t local_count;   /* outputs of the local reduction                    */
  int64_t global_count;  /* outputs after the exchange                         */
  int64_t out_offset;    /* where this rank's local result lands in out        */
  int64_t gang_offset;   /* first global gang index owned by this rank         */
} xr_shard_info;

/* Host-only: the exchange xr_reduce_sharded performs for this rank. */
int xr_shard_plan(int op, int dtype, const int64_t local_dims[3], unsigned level_mask,
                  int nranks, int rank, xr_shard_info* info);

/* NCCL unique id (128 bytes) on rank 0; broadcast it out of band
 * (torch.distributed in the Python binding). */
int xr_comm_get_unique_id(void* id128);
/* One communicator per process/GPU (device = CUDA ordinal used by this rank). */
int xr_comm_init(xr_comm_t* comm, int nranks, int rank, const void* id128, int device);
int xr_comm_destroy(xr_comm_t comm);

/* Fused exchange (default when set up): for whole-nest results (every level
 * reduced, or the kept ones of extent 1) the last CTA of the local reduction
 * writes its value into every peer's mailbox over NVLink (CUDA IPC, handles
 * all-gathered by xr_comm_init), publishes an epoch flag, waits for all ranks
 * and combines the values in rank order -- ONE kernel, no NCCL launch, the same
 * bits on every rank.  Set up at xr_comm_init if every peer can be mapped;
 * otherwise (or when disabled) the NCCL collectives below are used.  The wait
 * is bounded (20 s of %globaltimer; XR_EXCH_TIMEOUT_MS overrides): a rank
 * whose peers never arrive leaves out UNCHANGED and sets a host-mapped status
 * word, read by xr_comm_query without synchronising; while it is set, every
 * fused xr_reduce_sharded call returns XR_ERR_NCCL.
 * xr_comm_set_fused(comm, 0) switches this rank to the NCCL path (local, no
 * communication).  xr_comm_set_fused(comm, 1) is COLLECTIVE (every rank calls
 * it, nothing of the communicator in flight): it synchronises the device,
 * re-aligns the mailbox epochs across ranks (NCCL max), clears the status word
 * and enables the exchange; XR_ERR_UNSUPPORTED if a peer is not mapped. */
int xr_comm_set_fused(xr_comm_t comm, int enable);
int xr_comm_query(xr_comm_t comm, int* fused, int* status);

/* Local xr_reduce on this rank's gang slice + ONE collective on `stream`
 * (or the fused exchange above).  The collective runs at every world size,
 * including a 1-rank communicator.  Errors: as xr_reduce, XR_ERR_NCCL for an
 * NCCL failure or a timed-out fused exchange (see above). */
int xr_reduce_sharded(int op, int dtype, const int64_t local_dims[3], unsigned level_mask,
                      const void* in_local, void* out, xr_comm_t comm, xr_stream_t stream);

/* xr_reduce_sharded with HOST buffers: this rank's gang slice in_local_host
 * (host, pinned for the full PCIe rate) goes through the chunked H2D pipeline
 * of xr_reduce_host into a device partial, then the same collective as
 * xr_reduce_sharded (NCCL; the fused exchange needs a single-launch local
 * reduction and is not used here), and the GLOBAL result is copied to
 * out_host (host; global_count elements, also the init when
 * XR_INIT_FROM_OUT).  Synchronous.  Every rank calls it (NCCL rule). */
int xr_reduce_sharded_host(int op, int dtype, const int64_t local_dims[3], unsigned level_mask,
                           const void* in_local_host, void* out_host, xr_comm_t comm, xr_stream_t stream);

/* Single-device simulation of the fused exchange: nranks concurrent kernels on
 * separate streams, each reducing shards[r] into outs[r] (1 element) with its
 * own mailbox -- the real publish / spin / combine protocol.  Synchronous.
 * XR_ERR_NCCL if a rank never arrived (the waiting ranks leave their out
 * unchanged).  Test hooks: XR_TEST_SIM_SKIP_RANK=r never launches rank r;
 * XR_EXCH_TIMEOUT_MS bounds the wait (default 10 s here). */
int xr_reduce_fused_sim(int op, int dtype, const int64_t local_dims[3], unsigned level_mask,
                        const void* const* shards, int nranks, void* const* outs);

/* Single-device simulation of the sharded protocol (testing without NCCL):
 * shards[r] (DEVICE) holds rank r's slice; runs the nranks local reductions
 * and the same exchange semantics with device copies + the same fixed-order
 * combine kernel.  out as for rank 0 of xr_reduce_sharded. */
int xr_reduce_sharded_sim(int op, int dtype, const int64_t local_dims[3],
                          unsigned level_mask, const void* const* shards, int nranks,
                          void* out, xr_stream_t stream);

#ifdef __cplusplus
}
#endif
#endif /* XREDUCE_H */
