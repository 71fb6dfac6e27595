// xr_xform.cu -- SURVEY.md 8(f) N1: transform-reduce, the loop body before the
// reduction.  Two inputs x, y of the same nest:
//   XR_XF_DISK: Monte Carlo pi (Fig 13(c) @43561-44280, section 4
//     @42177-47503): count of x*x + y*y < 1, each operation rounded in the
//     inputs' type with __fmul_rn / __fadd_rn (no FMA, as the paper compiles,
//     @35389), so the predicate is decided exactly like the oracle; int64 out.
//   XR_XF_DOT: inner product (Fig 13(b) @41386-42177): sum of x*y, dtype out.
// Single pass like xr_reduce: private partials (16-B loads of BOTH inputs,
// 4+4 in flight), warp shuffles, CTA smem combine, last-CTA ticket.
// Canonical shapes R, KR, RKR (the seg decomposition), K, and the column
// shapes RK, KRK (xr_colunit.cuh: lanes own contiguous kept columns of BOTH
// inputs, warps stride the reduced rows, per-tile ticket).
#include <algorithm>
#include <cstdlib>

#include "../../include/xreduce.h"
#include "xr_internal.h"
#include "xr_ops.cuh"
#include "xr_colunit.cuh"

namespace xr {

int xform_workspace(cudaStream_t s, int64_t pbytes, int64_t ntick, void** partials, unsigned** tickets);

template <int XF, typename T> struct Xf;

template <typename T> struct Xf<XR_XF_DISK, T> {  // count of points inside the unit disk
  using Acc = unsigned long long;
  using Out = long long;
  static __device__ __forceinline__ Acc identity() { return 0ull; }
  static __device__ __forceinline__ Acc lift(T x, T y);
  static __device__ __forceinline__ Acc combine(Acc a, Acc b) { return a + b; }
  static __device__ __forceinline__ Acc lift_out(Out v) { return (Acc)v; }
  static __device__ __forceinline__ Out finish(Acc a) { return (Out)a; }
};
template <> __device__ __forceinline__ unsigned long long Xf<XR_XF_DISK, float>::lift(float x, float y) {
  return __fadd_rn(__fmul_rn(x, x), __fmul_rn(y, y)) < 1.0f ? 1ull : 0ull;
}
template <> __device__ __forceinline__ unsigned long long Xf<XR_XF_DISK, double>::lift(double x, double y) {
  return __dadd_rn(__dmul_rn(x, x), __dmul_rn(y, y)) < 1.0 ? 1ull : 0ull;
}

template <typename T> __device__ __forceinline__ T mul_rn(T a, T b) { return a * b; }
template <> __device__ __forceinline__ float mul_rn<float>(float a, float b) { return __fmul_rn(a, b); }
template <> __device__ __forceinline__ double mul_rn<double>(double a, double b) { return __dmul_rn(a, b); }

template <typename T> struct Xf<XR_XF_DOT, T> {  // inner product
  using B = Op<OP_ADD, T>;
  using Acc = typename B::Acc;
  using Out = T;
  static __device__ __forceinline__ Acc identity() { return B::identity(); }
  static __device__ __forceinline__ Acc lift(T x, T y) {
    if constexpr (IsFp<T>::value) return mul_rn(x, y);
    else return B::lift(x) * B::lift(y);  // unsigned: wraps mod 2^w (C6)
  }
  static __device__ __forceinline__ Acc combine(Acc a, Acc b) { return B::combine(a, b); }
  static __device__ __forceinline__ Acc lift_out(Out v) { return B::lift(v); }
  static __device__ __forceinline__ Out finish(Acc a) { return B::finish(a); }
};

template <typename X> __device__ __forceinline__ typename X::Acc xf_warp(typename X::Acc v) {
#pragma unroll
  for (int off = 16; off > 0; off >>= 1) v = X::combine(v, __shfl_xor_sync(0xffffffffu, v, off));
  return v;
}
template <typename X> __device__ __forceinline__ typename X::Acc xf_block(typename X::Acc v, typename X::Acc* smem) {
  v = xf_warp<X>(v);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (lane == 0) smem[warp] = v;
  __syncthreads();
  if (warp == 0) {
    v = lane < kBlock / 32 ? smem[lane] : X::identity();
    v = xf_warp<X>(v);
  }
  return v;
}

// Fold n elements of rows x, y into the lane's accumulators (group of W lanes).
template <typename X, typename T, int W, int U>
__device__ __forceinline__ void fold_row2(const T* __restrict__ x, const T* __restrict__ y, int64_t n, int lane,
                                          typename X::Acc (&acc)[U][16 / sizeof(T)]) {
  constexpr int VEC = 16 / sizeof(T);
  if ((((uintptr_t)x ^ (uintptr_t)y) & 15u) != 0) {  // different 16-B phase: scalar lanes
    for (int64_t i = lane; i < n; i += W) acc[0][0] = X::combine(acc[0][0], X::lift(__ldg(x + i), __ldg(y + i)));
    return;
  }
  int64_t head = (int64_t)((16u - ((uint32_t)(uintptr_t)x & 15u)) & 15u) / (int64_t)sizeof(T);
  if (head > n) head = n;
  if (lane < head) acc[0][0] = X::combine(acc[0][0], X::lift(__ldg(x + lane), __ldg(y + lane)));
  x += head;
  y += head;
  n -= head;
  const int64_t nv = n / VEC;
  const U128* __restrict__ xv = reinterpret_cast<const U128*>(x);
  const U128* __restrict__ yv = reinterpret_cast<const U128*>(y);
  int64_t v = lane;
  for (; v + (int64_t)(U - 1) * W < nv; v += (int64_t)U * W) {
    U128 a[U], b[U];
#pragma unroll
    for (int k = 0; k < U; ++k) {
      a[k] = ld_stream(xv + v + (int64_t)k * W);
      b[k] = ld_stream(yv + v + (int64_t)k * W);
    }
#pragma unroll
    for (int k = 0; k < U; ++k)
#pragma unroll
      for (int q = 0; q < VEC; ++q)
        acc[k][q] = X::combine(acc[k][q], X::lift(unpack<T>(a[k], q), unpack<T>(b[k], q)));
  }
  for (; v < nv; v += W) {
    const U128 a = ld_stream(xv + v), b = ld_stream(yv + v);
#pragma unroll
    for (int q = 0; q < VEC; ++q) acc[0][q] = X::combine(acc[0][q], X::lift(unpack<T>(a, q), unpack<T>(b, q)));
  }
  const int64_t tail = n - nv * VEC;
  if (lane < tail) acc[1 % U][0] = X::combine(acc[1 % U][0], X::lift(__ldg(x + nv * VEC + lane), __ldg(y + nv * VEC + lane)));
}

__device__ __forceinline__ int64_t xsplit(int64_t n, int64_t parts, int64_t i) {
  const int64_t q = n / parts, r = n % parts;
  return i * q + (i < r ? i : r);
}

// CTA-wide units, static round robin (deterministic), seg decomposition.
template <int XF, typename T>
__global__ void __launch_bounds__(kBlock) xform_kernel(SegArgs a, const void* in2) {
  pdl_wait();  // no global access above this line
  pdl_trigger();
  using X = Xf<XF, T>;
  using Acc = typename X::Acc;
  using Out = typename X::Out;
  constexpr int VEC = 16 / sizeof(T);
  constexpr int U = kUnroll;
  __shared__ Acc smem[32];
  __shared__ int s_last;
  Out* out = static_cast<Out*>(a.out);
  Acc* partials = static_cast<Acc*>(a.partials);
  const int64_t S = a.Sr * a.Sc;
  for (int64_t u = blockIdx.x; u < a.units; u += gridDim.x) {
    const int64_t o = u / S, s = u - o * S;
    const int64_t sr = s / a.Sc, sc = s - sr * a.Sc;
    const int64_t r0 = xsplit(a.C, a.Sr, sr), r1 = xsplit(a.C, a.Sr, sr + 1);
    const int64_t c0 = sc == 0 ? 0 : (xsplit(a.L, a.Sc, sc) / VEC) * VEC;
    const int64_t c1 = sc + 1 >= a.Sc ? a.L : (xsplit(a.L, a.Sc, sc + 1) / VEC) * VEC;
    Acc acc[U][VEC];
#pragma unroll
    for (int k = 0; k < U; ++k)
#pragma unroll
      for (int q = 0; q < VEC; ++q) acc[k][q] = X::identity();
    const int64_t base = o * a.oStride + c0;
    for (int64_t r = r0; r < r1; ++r) {
      const int64_t e = base + r * a.rowStride;
      fold_row2<X, T, kBlock, U>(static_cast<const T*>(a.in) + e, static_cast<const T*>(in2) + e, c1 - c0,
                                 threadIdx.x, acc);
    }
#pragma unroll
    for (int k = 1; k < U; ++k)
#pragma unroll
      for (int q = 0; q < VEC; ++q) acc[0][q] = X::combine(acc[0][q], acc[k][q]);
#pragma unroll
    for (int q = 1; q < VEC; ++q) acc[0][0] = X::combine(acc[0][0], acc[0][q]);
    Acc v = xf_block<X>(acc[0][0], smem);
    if (S == 1) {
      if (threadIdx.x == 0) {
        const Acc init = a.init_from_out ? X::lift_out(out[o]) : X::identity();
        out[o] = X::finish(X::combine(init, v));
      }
    } else {
      if (threadIdx.x == 0) {
        partials[u] = v;
        s_last = (ticket_add(&a.tickets[o]) == (unsigned)(S - 1));
      }
      __syncthreads();
      if (s_last) {
        __threadfence();
        Acc w = X::identity();
        for (int64_t i = threadIdx.x; i < S; i += kBlock) w = X::combine(w, __ldcg(partials + o * S + i));
        w = xf_block<X>(w, smem);
        if (threadIdx.x == 0) {
          const Acc init = a.init_from_out ? X::lift_out(out[o]) : X::identity();
          out[o] = X::finish(X::combine(init, w));
          a.tickets[o] = 0u;
        }
      }
    }
    __syncthreads();
  }
}

// Whole-array (R) shape on large, 16-B aligned inputs: the bulk-copy ring of
// the stream kernel (xr_kernels.cuh) for TWO inputs.  Each 16 KiB stage holds
// 8 KiB of x and the matching 8 KiB of y, streamed by the producer warp with
// cp.async.bulk (TMA engine) NS stages ahead across unit boundaries; the 8
// consumer warps apply the transform pairwise from shared memory.  Equal
// units claimed dynamically, one partial per unit folded in unit order by the
// last CTA (deterministic).  r01: the register path reached 0.84 / 0.88 of the
// copy peak on 2^27 / 2^28 Monte Carlo samples.
constexpr int kXfHalf = kStageBytes / 2;  // bytes of ONE input per stage
template <int XF, typename T, int NS>
__global__ void __launch_bounds__(kWsBlock, 3) xform_stream_kernel(const __grid_constant__ SegArgs a,
                                                                            const void* in2) {
  using X = Xf<XF, T>;
  using Acc = typename X::Acc;
  using Out = typename X::Out;
  constexpr int VEC = 16 / sizeof(T);
  constexpr int PER = kXfHalf / (16 * kConsThreads);  // 16-B vectors per consumer thread per input per stage
  constexpr int RING = 8;
  static_assert(PER >= 1, "stage geometry");
  extern __shared__ __align__(1024) unsigned char stage_mem[];  // NS * kStageBytes
  __shared__ __align__(8) uint64_t full[NS];
  __shared__ __align__(8) uint64_t empty[NS];
  __shared__ long long s_units[RING];
  __shared__ Acc smem[2][kConsWarps];
  __shared__ int s_last;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const T* __restrict__ xs = static_cast<const T*>(a.in);
  const T* __restrict__ ys = static_cast<const T*>(in2);
  Out* out = static_cast<Out*>(a.out);
  Acc* partials = static_cast<Acc*>(a.partials);
  const int64_t S = a.Sc;
  if (tid == 0) {
#pragma unroll
    for (int k = 0; k < NS; ++k) {
      mbar_init(&full[k], 1);
      mbar_init(&empty[k], kConsWarps);
    }
    fence_mbar_init();
  }
  __syncthreads();
  pdl_wait();  // no global access above this line
  pdl_trigger();
  auto range = [&](long long u, int64_t* c0, int64_t* nb, int64_t* c1) {
    *c0 = u == 0 ? 0 : (xsplit(a.L, S, u) / VEC) * VEC;
    *c1 = u + 1 >= S ? a.L : (xsplit(a.L, S, u + 1) / VEC) * VEC;
    *nb = ((*c1 - *c0) / VEC) * VEC;  // 16-B body (c0 is a multiple of VEC, the inputs 16-B aligned)
  };
  if (warp == 0) {  // ---------------- producer warp
    if (lane == 0) {
      int64_t g = 0;
      int seq = 0;
      long long u = claim_first(a.sched);
      while (true) {
        const long long nu = claim_next(a.sched);
        const int slot0 = (int)(g % NS);
        s_units[seq & (RING - 1)] = u < S ? u : -1;
        ++seq;
        if (u >= S) {
          if (g >= NS) mbar_wait(&empty[slot0], (unsigned)(((g / NS) - 1) & 1));
          mbar_arrive(&full[slot0]);
          break;
        }
        int64_t c0, nb, c1;
        range(u, &c0, &nb, &c1);
        const int64_t bytes = nb * (int64_t)sizeof(T);
        const int64_t nk = (bytes + kXfHalf - 1) / kXfHalf;
        for (int64_t k = 0; k < nk; ++k, ++g) {
          const int slot = (int)(g % NS);
          if (g >= NS) mbar_wait(&empty[slot], (unsigned)(((g / NS) - 1) & 1));
          const unsigned len = (unsigned)min((int64_t)kXfHalf, bytes - k * kXfHalf);
          mbar_expect_tx(&full[slot], 2 * len);
          const int64_t off = c0 * (int64_t)sizeof(T) + k * kXfHalf;
          bulk_g2s(stage_mem + slot * kStageBytes, reinterpret_cast<const char*>(xs) + off, len, &full[slot]);
          bulk_g2s(stage_mem + slot * kStageBytes + kXfHalf, reinterpret_cast<const char*>(ys) + off, len, &full[slot]);
        }
        u = nu;
      }
      sched_exit(a.sched);
    }
    return;
  }
  // ---------------- consumer warps
  const int ct = tid - 32, cw = warp - 1;
  int seq = 0;
  int64_t g = 0;
  Acc acc[PER][VEC];
#pragma unroll
  for (int j = 0; j < PER; ++j)
#pragma unroll
    for (int q = 0; q < VEC; ++q) acc[j][q] = X::identity();
  while (true) {
    mbar_wait(&full[g % NS], (unsigned)((g / NS) & 1));
    const long long u = s_units[seq & (RING - 1)];
    if (u < 0) break;
    int64_t c0, nb, c1;
    range(u, &c0, &nb, &c1);
    const int64_t tail = c1 - c0 - nb;  // last unit only: elements past the last 16-B vector
    if (ct < tail) acc[0][0] = X::combine(acc[0][0], X::lift(xs[c0 + nb + ct], ys[c0 + nb + ct]));
    const int64_t bytes = nb * (int64_t)sizeof(T);
    const int64_t nk = (bytes + kXfHalf - 1) / kXfHalf;
    for (int64_t k = 0; k < nk; ++k, ++g) {
      const int slot = (int)(g % NS);
      if (k > 0) mbar_wait(&full[slot], (unsigned)((g / NS) & 1));
      const int64_t len = min((int64_t)kXfHalf, bytes - k * kXfHalf);
      const unsigned char* st = stage_mem + slot * kStageBytes;
      U128 xv[PER], yv[PER];
#pragma unroll
      for (int j = 0; j < PER; ++j) {
        const int off = (ct + j * kConsThreads) * 16;
        if (len == kXfHalf || off < len) {
          xv[j] = *reinterpret_cast<const U128*>(st + off);
          yv[j] = *reinterpret_cast<const U128*>(st + kXfHalf + off);
        }
      }
#pragma unroll
      for (int j = 0; j < PER; ++j) {
        const int off = (ct + j * kConsThreads) * 16;
        if (len == kXfHalf || off < len) {
#pragma unroll
          for (int q = 0; q < VEC; ++q)
            acc[j][q] = X::combine(acc[j][q], X::lift(unpack<T>(xv[j], q), unpack<T>(yv[j], q)));
        }
      }
      fence_proxy_async_smem();  // generic reads before the async refill
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[slot]);
    }
    // the unit's partial: fixed-order fold of the accumulators, warp, consumers
    Acc v = acc[0][0];
#pragma unroll
    for (int j = 0; j < PER; ++j)
#pragma unroll
      for (int q = 0; q < VEC; ++q) {
        if (j || q) v = X::combine(v, acc[j][q]);
        acc[j][q] = X::identity();
      }
    v = xf_warp<X>(v);
    if (lane == 0) smem[seq & 1][cw] = v;
    cons_sync();
    if (ct == 0) {
      Acc w = X::identity();
#pragma unroll
      for (int k = 0; k < kConsWarps; ++k) w = X::combine(w, smem[seq & 1][k]);
      partials[u] = w;
    }
    ++seq;
  }
  // a4: one ticket per CTA; the last CTA folds the S unit partials in unit order
  if (ct == 0) s_last = (ticket_add(&a.tickets[0]) == gridDim.x - 1u);
  cons_sync();
  if (s_last) {
    __threadfence();
    Acc w = X::identity();
    for (int64_t i = ct; i < S; i += kConsThreads) w = X::combine(w, __ldcg(partials + i));
    w = xf_warp<X>(w);
    if (lane == 0) smem[0][cw] = w;
    cons_sync();
    if (ct == 0) {
      Acc z = X::identity();
#pragma unroll
      for (int k = 0; k < kConsWarps; ++k) z = X::combine(z, smem[0][k]);
      const Acc init = a.init_from_out ? X::lift_out(out[0]) : X::identity();
      out[0] = X::finish(X::combine(init, z));
      a.tickets[0] = 0u;
    }
  }
}

template <int XF, typename T>
__global__ void __launch_bounds__(kBlock) xform_ident_kernel(EltArgs a, const void* in2) {
  pdl_wait();  // no global access above this line
  pdl_trigger();
  using X = Xf<XF, T>;
  using Out = typename X::Out;
  Out* out = static_cast<Out*>(a.out);
  const T* x = static_cast<const T*>(a.in);
  const T* y = static_cast<const T*>(in2);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < a.n; i += (int64_t)gridDim.x * blockDim.x) {
    const typename X::Acc init = a.init_from_out ? X::lift_out(out[i]) : X::identity();
    out[i] = X::finish(X::combine(init, a.in ? X::lift(x[i], y[i]) : X::identity()));
  }
}

// Column shapes (RK, KRK): CTA-wide column units, static round robin.
template <int XF, typename T, int VEC>
__global__ void __launch_bounds__(kBlock) xform_col_kernel(const __grid_constant__ ColArgs a, const void* in2) {
  pdl_wait();  // no global access above this line
  pdl_trigger();
  using X = Xf<XF, T>;
  __shared__ __align__(16) unsigned char sm[col_unit_smem<X, VEC>()];
  __shared__ int s_last;
  for (int64_t u = blockIdx.x; u < a.units; u += gridDim.x)
    col_unit<X, T, 2, VEC, kUnroll>(a, static_cast<const T*>(a.in), static_cast<const T*>(in2), u, sm, &s_last);
}

template <int XF, typename T, int VEC>
static cudaError_t xform_col_launch(const ColArgs& c, const void* in2, int sms, cudaStream_t s) {
  const int occ = occ_dev<xform_col_kernel<XF, T, VEC>>(kBlock, 0);
  return launch_pdl(xform_col_kernel<XF, T, VEC>, dim3((unsigned)grid_for(c.units, sms, occ)), dim3(kBlock), 0, s, c, in2);
}

template <int XF, typename T>
static cudaError_t xform_stream_launch(const SegArgs& sa, const void* in2, int sms, cudaStream_t s) {
  auto kern = xform_stream_kernel<XF, T, kStages>;
  constexpr int dyn = kStages * kStageBytes;
  const int occ = occ_dev<xform_stream_kernel<XF, T, kStages>>(kWsBlock, dyn);
  const cudaError_t e = launch_pdl(kern, dim3((unsigned)grid_for(sa.units, sms, occ)), dim3(kWsBlock), dyn, s, sa, in2);
  count_launch();
  return e != cudaSuccess ? e : cudaPeekAtLastError();
}

template <int XF, typename T>
static cudaError_t xform_launch(Plan& p, const void* in2, int sms, cudaStream_t s) {
  cudaError_t le = cudaSuccess;
  if (p.kernel == K_FILL || p.kernel == K_IDENT) {
    EltArgs e = p.elt;
    if (p.kernel == K_FILL) e.in = nullptr;
    const int64_t grid = grid_for((e.n + kBlock - 1) / kBlock, sms, 8);
    le = launch_pdl(xform_ident_kernel<XF, T>, dim3((unsigned)grid), dim3(kBlock), 0, s, e, in2);
  } else if (p.kernel == K_COL) {
    if (p.vec > 1) le = xform_col_launch<XF, T, 16 / sizeof(T)>(p.col, in2, sms, s);
    else le = xform_col_launch<XF, T, 1>(p.col, in2, sms, s);
  } else {
    const int occ = occ_dev<xform_kernel<XF, T>>(kBlock, 0);
    le = launch_pdl(xform_kernel<XF, T>, dim3((unsigned)grid_for(p.units, sms, occ)), dim3(kBlock), 0, s, p.seg, in2);
  }
  count_launch();
  return le != cudaSuccess ? le : cudaPeekAtLastError();
}

}  // namespace xr

using namespace xr;

extern "C" int xr_transform_reduce(int xform, int dtype, const int64_t nest_dims[3], unsigned level_mask,
                                   const void* x, const void* y, void* out, xr_stream_t stream) {
  if (xform != XR_XF_DISK && xform != XR_XF_DOT) return XR_ERR_INVALID;
  if (dtype < XR_INT32 || dtype > XR_FP64 || !nest_dims) return XR_ERR_INVALID;
  if (xform == XR_XF_DISK && dtype != XR_FP32 && dtype != XR_FP64) return XR_ERR_UNSUPPORTED;
  if ((level_mask & 7u) == 0u || (level_mask & ~(7u | XR_INIT_FROM_OUT)) != 0u) return XR_ERR_INVALID;
  int64_t total = 1, count = 1;
  for (int d = 0; d < 3; ++d) {
    if (nest_dims[d] < 0) return XR_ERR_INVALID;
    if (nest_dims[d] != 0 && total > (INT64_MAX / 8) / nest_dims[d]) return XR_ERR_INVALID;
    total *= nest_dims[d];
    if (!((level_mask >> d) & 1u)) count *= nest_dims[d];
  }
  if (count == 0) return XR_OK;
  const int size = dtype_size(dtype), osize = xform == XR_XF_DISK ? 8 : size;
  if (!out || (total > 0 && (!x || !y))) return XR_ERR_INVALID;
  if (((uintptr_t)out % osize) || (total > 0 && (((uintptr_t)x % size) || ((uintptr_t)y % size))))
    return XR_ERR_INVALID;
  Plan p;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return XR_ERR_CUDA; }
  int sms = 148;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  // whole-array transform-reduce of large 16-B aligned inputs: the bulk ring
  {
    bool whole = true;
    for (int d = 0; d < 3; ++d)
      if (!((level_mask >> d) & 1u) && nest_dims[d] != 1) whole = false;
    const bool al = ((uintptr_t)x % 16 == 0) && ((uintptr_t)y % 16 == 0);
    if (whole && al && total * size >= kSmallBytes && std::getenv("XR_NO_BULK") == nullptr &&
        std::getenv("XR_NO_XF_STREAM") == nullptr) {
      // equal units, ~8 per resident CTA (3 per SM), each >= 4 stages of either input
      const int64_t cap = (int64_t)sms * 3;
      const int64_t S = std::max<int64_t>(1, std::min<int64_t>(8 * cap, total * size / (4 * kXfHalf)));
      void* partials = nullptr;
      unsigned* tickets = nullptr;
      int st = xform_workspace((cudaStream_t)stream, S * 8, 2 + 4, &partials, &tickets);
      if (st) return st;
      SegArgs sa{};
      sa.in = x; sa.out = out; sa.partials = partials; sa.tickets = tickets;
      sa.sched = reinterpret_cast<unsigned long long*>(tickets + 2);
      sa.O = 1; sa.C = 1; sa.L = total; sa.Sr = 1; sa.Sc = S; sa.units = S;
      sa.init_from_out = (level_mask & XR_INIT_FROM_OUT) ? 1 : 0;
      cudaStream_t s = (cudaStream_t)stream;
      cudaError_t e;
      if (xform == XR_XF_DISK) {
        e = dtype == XR_FP32 ? xform_stream_launch<XR_XF_DISK, float>(sa, y, sms, s)
                             : xform_stream_launch<XR_XF_DISK, double>(sa, y, sms, s);
      } else {
        switch (dtype) {
          case XR_INT32: e = xform_stream_launch<XR_XF_DOT, int32_t>(sa, y, sms, s); break;
          case XR_INT64: e = xform_stream_launch<XR_XF_DOT, int64_t>(sa, y, sms, s); break;
          case XR_FP32: e = xform_stream_launch<XR_XF_DOT, float>(sa, y, sms, s); break;
          default: e = xform_stream_launch<XR_XF_DOT, double>(sa, y, sms, s); break;
        }
      }
      if (e != cudaSuccess) { cudaGetLastError(); return XR_ERR_CUDA; }
      return XR_OK;
    }
  }
  // in_addr: the column path takes 16-B vectors only if BOTH inputs are aligned
  make_plan(xform == XR_XF_DOT ? XR_OP_ADD : XR_OP_LOR /* non-chain-capped */, dtype, nest_dims, level_mask & 7u,
            (uint64_t)((uintptr_t)x | (uintptr_t)y), sms, &p, /*seg_only=*/true);
  if (p.kernel == K_NONE) return XR_OK;
  // partial slots sized for the transform's accumulator (DISK: 8-byte counts)
  const int64_t pslots = p.kernel == K_COL ? p.col.B * p.col.tiles * p.col.S * 32 * p.vec : p.units;
  const int64_t pbytes = p.splits > 1 ? pslots * 8 : 0;
  void* partials = nullptr;
  unsigned* tickets = nullptr;
  int st = xform_workspace((cudaStream_t)stream, pbytes, p.tickets, &partials, &tickets);
  if (st) return st;
  const int ifo = (level_mask & XR_INIT_FROM_OUT) ? 1 : 0;
  p.seg.in = x; p.seg.out = out; p.seg.partials = partials; p.seg.tickets = tickets; p.seg.init_from_out = ifo;
  p.col.in = x; p.col.out = out; p.col.partials = partials; p.col.tickets = tickets; p.col.init_from_out = ifo;
  p.elt.in = x; p.elt.out = out; p.elt.init_from_out = ifo;
  cudaStream_t s = (cudaStream_t)stream;
  cudaError_t e;
  if (xform == XR_XF_DISK) {
    e = dtype == XR_FP32 ? xform_launch<XR_XF_DISK, float>(p, y, sms, s) : xform_launch<XR_XF_DISK, double>(p, y, sms, s);
  } else {
    switch (dtype) {
      case XR_INT32: e = xform_launch<XR_XF_DOT, int32_t>(p, y, sms, s); break;
      case XR_INT64: e = xform_launch<XR_XF_DOT, int64_t>(p, y, sms, s); break;
      case XR_FP32: e = xform_launch<XR_XF_DOT, float>(p, y, sms, s); break;
      default: e = xform_launch<XR_XF_DOT, double>(p, y, sms, s); break;
    }
  }
  if (e != cudaSuccess) { cudaGetLastError(); return XR_ERR_CUDA; }
  return XR_OK;
}
