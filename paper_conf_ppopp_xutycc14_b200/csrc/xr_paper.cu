// xr_paper.cu -- SURVEY.md 8(f) N3: the paper's OWN code-generation scheme,
// written for sm_100a as an in-house A/B baseline (there are no comparison
// systems to run: OpenUH / PGI / CAPS are unavailable).  It follows PAPER.md:
//  - launch: gang = blockIdx.x, worker = threadIdx.y, vector = threadIdx.x
//    (@11499-11699, Table 1); num_gangs x (vector_length x num_workers), by
//    default the paper's 192 x (128 x 8) (@35893-36486);
//  - loops: Fig 3 (@13404) -- each level starts at its thread index and
//    strides by its thread count ("window sliding", @25875-26664);
//  - vector tier: private partial, then the interleaved log-step over a
//    shared-memory row laid out like global memory (Fig 6c, Fig 7,
//    @19949-21328); worker tier: log-step over the workers of a column
//    (Fig 8c idea, @23603-24615);
//  - gang tier: partial[] in global memory plus a SECOND kernel launch that
//    reduces it in one block (Fig 5c, @24887-25280); RMP with gang involved:
//    a global buffer of every reducing thread + second kernel (@28433-29414,
//    @30925-31587).
// Deviations needed to run correctly on sm_70+: the log-step's last 6 steps
// use __syncwarp() (warp-synchronous code without it is a data race on
// independent-thread-scheduling GPUs), and loops whose trip count differs
// between threads of a block are padded so every thread reaches each
// __syncthreads() (Fig 5a has a barrier inside while(j), a divergence hazard
// when NJ % blockDim.y != 0).  Supported: masks g, w, v (Table 2's
// single-level positions) and the paper's three RMP scenarios (3.2.1
// @28973-29561: gang & worker, gang & worker & vector, worker & vector; gang &
// vector "cannot span ... without going through the worker" and stays
// unsupported), ops + * max, dtypes int32 fp32 fp64 (Table 2's Int / Float /
// Double).
#include <algorithm>

#include "../../include/xreduce.h"
#include "xr_internal.h"
#include "xr_ops.cuh"

namespace xr {

int paper_workspace(cudaStream_t s, int64_t bytes, void** buf);

// Interleaved log-step over n (power of two) values at stride `st` in shared
// memory: value index t combines t + s for s = n/2 .. 1 (Fig 7).  Threads with
// t >= s idle.  Barriers: __syncthreads between steps while s > 32 (threads
// of different warps), __syncwarp below.
template <typename O>
__device__ __forceinline__ void logstep(typename O::Acc* sbuf, int t, int n, int st, bool same_warp_tail) {
  for (int s = n / 2; s > 0; s >>= 1) {
    if (t < s) sbuf[t * st] = O::combine(sbuf[t * st], sbuf[(t + s) * st]);
    if (s > 32 || !same_warp_tail) __syncthreads();
    else __syncwarp();
  }
}

// ---- mask v: out[k][j] = init (+) sum_i in[k][j][i]  (Fig 4a / 5a)
template <int OP, typename T>
__global__ void paper_vector_kernel(const T* in, T* out, int64_t NK, int64_t NJ, int64_t NI, int ifo) {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  extern __shared__ unsigned char sraw[];
  Acc* sbuf = reinterpret_cast<Acc*>(sraw);
  const int tx = threadIdx.x, ty = threadIdx.y, bdx = blockDim.x, bdy = blockDim.y;
  for (int64_t k = blockIdx.x; k < NK; k += gridDim.x) {
    const int64_t jtrips = (NJ + bdy - 1) / bdy;  // padded: every thread reaches the barriers
    for (int64_t jt = 0; jt < jtrips; ++jt) {
      const int64_t j = ty + jt * bdy;
      Acc priv = O::identity();  // i_sum_priv = 0
      if (j < NJ)
        for (int64_t i = tx; i < NI; i += bdx) priv = O::combine(priv, O::lift(in[(k * NJ + j) * NI + i]));
      sbuf[tx + ty * bdx] = priv;  // row layout = global layout (Fig 6c)
      __syncthreads();
      logstep<O>(sbuf + ty * bdx, tx, bdx, 1, true);  // reduce_vector(sbuf, j)
      if (tx == 0 && j < NJ) {
        const int64_t o = k * NJ + j;
        const Acc init = ifo ? O::lift(out[o]) : O::identity();  // original value after the tree
        out[o] = O::finish(O::combine(init, sbuf[ty * bdx]));
      }
      __syncthreads();
    }
  }
}

// ---- mask w: out[k][i] = init (+) sum_j in[k][j][i]  (Fig 4b / 8c, all i)
template <int OP, typename T>
__global__ void paper_worker_kernel(const T* in, T* out, int64_t NK, int64_t NJ, int64_t NI, int ifo) {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  extern __shared__ unsigned char sraw[];
  Acc* sbuf = reinterpret_cast<Acc*>(sraw);
  const int tx = threadIdx.x, ty = threadIdx.y, bdx = blockDim.x, bdy = blockDim.y;
  for (int64_t k = blockIdx.x; k < NK; k += gridDim.x) {
    const int64_t itrips = (NI + bdx - 1) / bdx;
    for (int64_t it = 0; it < itrips; ++it) {
      const int64_t i = tx + it * bdx;
      Acc priv = O::identity();  // j_sum_priv = 0
      if (i < NI)
        for (int64_t j = ty; j < NJ; j += bdy) priv = O::combine(priv, O::lift(in[(k * NJ + j) * NI + i]));
      sbuf[tx + ty * bdx] = priv;
      __syncthreads();
      logstep<O>(sbuf + tx, ty, bdy, bdx, false);  // the workers of column tx
      if (ty == 0 && i < NI) {
        const int64_t o = k * NI + i;
        const Acc init = ifo ? O::lift(out[o]) : O::identity();
        out[o] = O::finish(O::combine(init, sbuf[tx]));
      }
      __syncthreads();
    }
  }
}

// ---- mask g, first launch: partial[gang][j][i] (Fig 5c, one value per output)
template <int OP, typename T>
__global__ void paper_gang_partial_kernel(const T* in, typename Op<OP, T>::Acc* partial, int64_t NK, int64_t NJ,
                                          int64_t NI) {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  for (int64_t j = threadIdx.y; j < NJ; j += blockDim.y)
    for (int64_t i = threadIdx.x; i < NI; i += blockDim.x) {
      Acc priv = O::identity();  // sum_priv, private for each gang
      for (int64_t k = blockIdx.x; k < NK; k += gridDim.x) priv = O::combine(priv, O::lift(in[(k * NJ + j) * NI + i]));
      partial[(int64_t)blockIdx.x * NJ * NI + j * NI + i] = priv;
    }
}

// ---- second launch: reduce `rows` partials per output in one block per
// output chunk with the log-step ("the same reduction kernel as the one in
// vector", @25084-25280).  buf layout [rows][nout].
template <int OP, typename T>
__global__ void paper_second_kernel(const typename Op<OP, T>::Acc* buf, int64_t rows, int64_t nout, T* out, int ifo) {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  extern __shared__ unsigned char sraw[];
  Acc* sbuf = reinterpret_cast<Acc*>(sraw);
  const int t = threadIdx.x, n = blockDim.x;
  for (int64_t o = blockIdx.x; o < nout; o += gridDim.x) {
    Acc priv = O::identity();
    for (int64_t r = t; r < rows; r += n) priv = O::combine(priv, buf[r * nout + o]);
    sbuf[t] = priv;
    __syncthreads();
    logstep<O>(sbuf, t, n, 1, true);
    if (t == 0) {
      const Acc init = ifo ? O::lift(out[o]) : O::identity();
      out[o] = O::finish(O::combine(init, sbuf[0]));
    }
    __syncthreads();
  }
}

// ---- mask gwv, first launch: RMP buffer of every reducing thread
// (gangs x workers x vectors, @30925-31587); the whole nest as one window.
template <int OP, typename T>
__global__ void paper_rmp_kernel(const T* in, typename Op<OP, T>::Acc* buf, int64_t N) {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  const int64_t tid = ((int64_t)blockIdx.x * blockDim.y + threadIdx.y) * blockDim.x + threadIdx.x;
  const int64_t nth = (int64_t)gridDim.x * blockDim.y * blockDim.x;
  Acc priv = O::identity();
  for (int64_t e = tid; e < N; e += nth) priv = O::combine(priv, O::lift(in[e]));
  buf[tid] = priv;
}

// ---- mask wv (RMP worker & vector, 3.2.1): the buffer of every reducing
// thread (workers x vectors) lives in SHARED memory ("the buffer is stored in
// the shared memory. Each thread writes its own partial reduction result into
// this buffer and continues the reduction operation in the shared memory",
// @28690-28973); one log-step over all of it per gang iteration k.
template <int OP, typename T>
__global__ void paper_wv_kernel(const T* in, T* out, int64_t NK, int64_t NJ, int64_t NI, int ifo) {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  extern __shared__ unsigned char sraw[];
  Acc* sbuf = reinterpret_cast<Acc*>(sraw);
  const int tx = threadIdx.x, ty = threadIdx.y, bdx = blockDim.x, bdy = blockDim.y;
  const int t = ty * bdx + tx, n = bdx * bdy;
  for (int64_t k = blockIdx.x; k < NK; k += gridDim.x) {
    Acc priv = O::identity();
    for (int64_t j = ty; j < NJ; j += bdy)        // worker loop
      for (int64_t i = tx; i < NI; i += bdx)      // vector loop
        priv = O::combine(priv, O::lift(in[(k * NJ + j) * NI + i]));
    sbuf[t] = priv;  // unique id of the thread
    __syncthreads();
    logstep<O>(sbuf, t, n, 1, true);
    if (t == 0) {
      const Acc init = ifo ? O::lift(out[k]) : O::identity();
      out[k] = O::finish(O::combine(init, sbuf[0]));
    }
    __syncthreads();
  }
}

// ---- mask gw (RMP gang & worker, 3.2.1), first launch: a GLOBAL buffer of
// every reducing thread (gangs x workers) per kept vector iteration i ("the
// buffer is allocated in the global memory since the reduction spans across
// gangs", @29217-29414); layout [gang][worker][NI].  The second launch is
// paper_second_kernel over rows = gangs * workers.
template <int OP, typename T>
__global__ void paper_gw_partial_kernel(const T* in, typename Op<OP, T>::Acc* buf, int64_t NK, int64_t NJ,
                                        int64_t NI) {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  const int64_t row = (int64_t)blockIdx.x * blockDim.y + threadIdx.y;
  for (int64_t i = threadIdx.x; i < NI; i += blockDim.x) {  // vector loop (kept)
    Acc priv = O::identity();
    for (int64_t k = blockIdx.x; k < NK; k += gridDim.x)    // gang loop
      for (int64_t j = threadIdx.y; j < NJ; j += blockDim.y)  // worker loop
        priv = O::combine(priv, O::lift(in[(k * NJ + j) * NI + i]));
    buf[row * NI + i] = priv;
  }
}

template <int OP, typename T>
static int paper_typed(const int64_t* d, unsigned mask, const T* in, T* out, int gangs, int workers, int vector,
                       cudaStream_t s) {
  using Acc = typename Op<OP, T>::Acc;
  const int ifo = (mask & XR_INIT_FROM_OUT) ? 1 : 0;
  const dim3 block(vector, workers);
  const size_t sb = (size_t)vector * workers * sizeof(Acc);
  switch (mask & 7u) {
    case XR_VECTOR:
      paper_vector_kernel<OP, T><<<gangs, block, sb, s>>>(in, out, d[0], d[1], d[2], ifo);
      count_launch();
      break;
    case XR_WORKER:
      paper_worker_kernel<OP, T><<<gangs, block, sb, s>>>(in, out, d[0], d[1], d[2], ifo);
      count_launch();
      break;
    case XR_GANG: {
      void* buf = nullptr;
      const int64_t nout = d[1] * d[2];
      int st = paper_workspace(s, (int64_t)gangs * nout * sizeof(Acc), &buf);
      if (st) return st;
      paper_gang_partial_kernel<OP, T><<<gangs, block, 0, s>>>(in, (Acc*)buf, d[0], d[1], d[2]);
      count_launch();
      const int nb = 256;
      paper_second_kernel<OP, T><<<(unsigned)std::min<int64_t>(nout, 65535), nb, nb * sizeof(Acc), s>>>(
          (const Acc*)buf, gangs, nout, out, ifo);
      count_launch();
      break;
    }
    case XR_WORKER | XR_VECTOR:
      paper_wv_kernel<OP, T><<<gangs, block, sb, s>>>(in, out, d[0], d[1], d[2], ifo);
      count_launch();
      break;
    case XR_GANG | XR_WORKER: {
      void* buf = nullptr;
      const int64_t rows = (int64_t)gangs * workers, nout = d[2];
      int st = paper_workspace(s, rows * nout * sizeof(Acc), &buf);
      if (st) return st;
      paper_gw_partial_kernel<OP, T><<<gangs, block, 0, s>>>(in, (Acc*)buf, d[0], d[1], d[2]);
      count_launch();
      const int nb = 256;
      paper_second_kernel<OP, T><<<(unsigned)std::min<int64_t>(nout, 65535), nb, nb * sizeof(Acc), s>>>(
          (const Acc*)buf, rows, nout, out, ifo);
      count_launch();
      break;
    }
    case 7u: {
      void* buf = nullptr;
      const int64_t nth = (int64_t)gangs * workers * vector;
      int st = paper_workspace(s, nth * sizeof(Acc), &buf);
      if (st) return st;
      paper_rmp_kernel<OP, T><<<gangs, block, 0, s>>>(in, (Acc*)buf, d[0] * d[1] * d[2]);
      count_launch();
      paper_second_kernel<OP, T><<<1, 1024, 1024 * sizeof(Acc), s>>>((const Acc*)buf, nth, 1, out, ifo);
      count_launch();
      break;
    }
    default:
      return XR_ERR_UNSUPPORTED;
  }
  if (cudaPeekAtLastError() != cudaSuccess) { cudaGetLastError(); return XR_ERR_CUDA; }
  return XR_OK;
}

}  // namespace xr

using namespace xr;

extern "C" int xr_reduce_paper(int op, int dtype, const int64_t nest_dims[3], unsigned level_mask, const void* in,
                               void* out, int num_gangs, int num_workers, int vector_length, xr_stream_t stream) {
  if (!nest_dims || (level_mask & ~(7u | XR_INIT_FROM_OUT)) != 0u) return XR_ERR_INVALID;
  const unsigned m = level_mask & 7u;
  if (m == (XR_GANG | XR_VECTOR) || m == 0u) return XR_ERR_UNSUPPORTED;  // gang & vector: not in the paper
  if (op != XR_OP_ADD && op != XR_OP_MUL && op != XR_OP_MAX) return XR_ERR_UNSUPPORTED;
  if (dtype != XR_INT32 && dtype != XR_FP32 && dtype != XR_FP64) return XR_ERR_UNSUPPORTED;
  for (int d = 0; d < 3; ++d)
    if (nest_dims[d] < 1) return XR_ERR_INVALID;
  if (num_gangs <= 0) num_gangs = 192;      // 12 SMs x 16 blocks (@36240-36486)
  if (num_workers <= 0) num_workers = 8;    // 1024-thread block limit
  if (vector_length <= 0) vector_length = 128;
  if ((vector_length & (vector_length - 1)) || (num_workers & (num_workers - 1)) ||
      vector_length * num_workers > 1024 || vector_length < 32)
    return XR_ERR_INVALID;  // the log-step wants powers of two (@33355-34930)
  if (!in || !out) return XR_ERR_INVALID;
  cudaStream_t s = (cudaStream_t)stream;
#define XR_PAPER_CASE(OPC, T)                                                                                     \
  return paper_typed<OPC, T>(nest_dims, level_mask, static_cast<const T*>(in), static_cast<T*>(out), num_gangs,  \
                             num_workers, vector_length, s)
  switch (dtype * 16 + op) {
    case XR_INT32 * 16 + XR_OP_ADD: XR_PAPER_CASE(OP_ADD, int32_t);
    case XR_INT32 * 16 + XR_OP_MUL: XR_PAPER_CASE(OP_MUL, int32_t);
    case XR_INT32 * 16 + XR_OP_MAX: XR_PAPER_CASE(OP_MAX, int32_t);
    case XR_FP32 * 16 + XR_OP_ADD: XR_PAPER_CASE(OP_ADD, float);
    case XR_FP32 * 16 + XR_OP_MUL: XR_PAPER_CASE(OP_MUL, float);
    case XR_FP32 * 16 + XR_OP_MAX: XR_PAPER_CASE(OP_MAX, float);
    case XR_FP64 * 16 + XR_OP_ADD: XR_PAPER_CASE(OP_ADD, double);
    case XR_FP64 * 16 + XR_OP_MUL: XR_PAPER_CASE(OP_MUL, double);
    default: XR_PAPER_CASE(OP_MAX, double);
  }
#undef XR_PAPER_CASE
}
