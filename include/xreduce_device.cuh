// include/xreduce_device.cuh -- the device-callable half of the xreduce
// boundary: the operator traits and the reduction tiers
// the library's own kernels use, for fusing a reduction into a user kernel.
// Header-only CUDA C++ for sm_100a (nvcc -std=c++17).
//
// Tier mapping:
//   a1 private partials : identity-initialised register accumulators, the
//                         paper's "each vector thread first creates a private
//                         variable and does the partial reduction itself"
//                         (PAPER.md @19558-19752, 3.1.1; Fig 5 i_sum_priv).
//   a2 vector tier      : group_reduce -- intra-warp combine with REDUX / VOTE /
//                         SHFL instead of the shared-memory interleaved
//                         log-step of Fig 7 (@19365-21328).
//   a3 worker tier      : block_reduce -- cross-warp combine through <= 32
//                         shared-memory slots and one barrier, cf. Fig 8(c)
//                         (@23603-24615).
//   a4 gang tier        : grid_reduce_gmem -- the shared-memory-free variant:
//                         warp partials in global memory and a last-warp-done
//                         ticket, for kernels that reserve all shared memory
//                         ("the shared memory is sometimes reserved for other
//                         computation ... we would need to move the reduction
//                         operation to the global memory", @32570-33355).
// All operators are associative and commutative, so any combine order is
// licensed (@15024-15239, 3); fixed layouts make the order deterministic.
//
// Usage (device code):
//   using O = xr::Op<xr::OP_ADD, float>;      // identity / lift / combine / finish
//   O::Acc v = O::identity(); ... v = O::combine(v, O::lift(x));
//   v = xr::group_reduce<xr::OP_ADD, float, 32>(v);              // whole warp
//   v = xr::block_reduce<xr::OP_ADD, float, 256>(v, slots32);    // warp 0 valid
//   xr::grid_reduce_gmem<xr::OP_ADD, float>(v, ws, out);         // no smem
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace xr {

enum : int { OP_ADD = 0, OP_MUL = 1, OP_MAX = 2, OP_MIN = 3, OP_BAND = 4,
             OP_BOR = 5, OP_BXOR = 6, OP_LAND = 7, OP_LOR = 8 };

template <typename T> struct Unsigned;
template <> struct Unsigned<int32_t> { using type = uint32_t; };
template <> struct Unsigned<int64_t> { using type = uint64_t; };

template <typename T> struct IsFp { static constexpr bool value = false; };
template <> struct IsFp<float> { static constexpr bool value = true; };
template <> struct IsFp<double> { static constexpr bool value = true; };

template <typename T> __device__ __forceinline__ T lowest();
template <> __device__ __forceinline__ int32_t lowest<int32_t>() { return INT32_MIN; }
template <> __device__ __forceinline__ int64_t lowest<int64_t>() { return INT64_MIN; }
template <> __device__ __forceinline__ float lowest<float>() { return __int_as_float(0xff800000u); }
template <> __device__ __forceinline__ double lowest<double>() { return __longlong_as_double(0xfff0000000000000ull); }
template <typename T> __device__ __forceinline__ T highest();
template <> __device__ __forceinline__ int32_t highest<int32_t>() { return INT32_MAX; }
template <> __device__ __forceinline__ int64_t highest<int64_t>() { return INT64_MAX; }
template <> __device__ __forceinline__ float highest<float>() { return __int_as_float(0x7f800000u); }
template <> __device__ __forceinline__ double highest<double>() { return __longlong_as_double(0x7ff0000000000000ull); }


// Op traits.  Acc is the accumulator type:
//   int  + * & | ^ : unsigned of the same width (two's-complement wrap, C6)
//   int  max min   : the signed type
//   fp   + * max min : the type itself (C23: accumulate in dtype)
//   && ||          : uint32, nonzero = true (C8; see Logical)
template <int OP, typename T, bool FP = IsFp<T>::value> struct Op;

// ---- integers: + * & | ^
template <int OP, typename T> struct IntArith {
  using Acc = typename Unsigned<T>::type;
  static __device__ __forceinline__ Acc identity() {
    return OP == OP_MUL ? Acc(1) : OP == OP_BAND ? ~Acc(0) : Acc(0);
  }
  static __device__ __forceinline__ Acc lift(T x) { return static_cast<Acc>(x); }
  static __device__ __forceinline__ Acc combine(Acc a, Acc b) {
    if constexpr (OP == OP_ADD) return a + b;
    else if constexpr (OP == OP_MUL) return a * b;
    else if constexpr (OP == OP_BAND) return a & b;
    else if constexpr (OP == OP_BOR) return a | b;
    else return a ^ b;
  }
  static __device__ __forceinline__ T finish(Acc a) { return static_cast<T>(a); }
};
template <typename T> struct Op<OP_ADD, T, false> : IntArith<OP_ADD, T> {};
template <typename T> struct Op<OP_MUL, T, false> : IntArith<OP_MUL, T> {};
template <typename T> struct Op<OP_BAND, T, false> : IntArith<OP_BAND, T> {};
template <typename T> struct Op<OP_BOR, T, false> : IntArith<OP_BOR, T> {};
template <typename T> struct Op<OP_BXOR, T, false> : IntArith<OP_BXOR, T> {};

// ---- integers: max min
template <typename T> struct Op<OP_MAX, T, false> {
  using Acc = T;
  static __device__ __forceinline__ Acc identity() { return lowest<T>(); }
  static __device__ __forceinline__ Acc lift(T x) { return x; }
  static __device__ __forceinline__ Acc combine(Acc a, Acc b) { return a > b ? a : b; }
  static __device__ __forceinline__ T finish(Acc a) { return a; }
};
template <typename T> struct Op<OP_MIN, T, false> {
  using Acc = T;
  static __device__ __forceinline__ Acc identity() { return highest<T>(); }
  static __device__ __forceinline__ Acc lift(T x) { return x; }
  static __device__ __forceinline__ Acc combine(Acc a, Acc b) { return a < b ? a : b; }
  static __device__ __forceinline__ T finish(Acc a) { return a; }
};

// ---- floating point: + *   (identity +0.0 / 1.0; reading C4)
template <typename T> struct Op<OP_ADD, T, true> {
  using Acc = T;
  static __device__ __forceinline__ Acc identity() { return T(0); }
  static __device__ __forceinline__ Acc lift(T x) { return x; }
  static __device__ __forceinline__ Acc combine(Acc a, Acc b) { return a + b; }
  static __device__ __forceinline__ T finish(Acc a) { return a; }
};
template <typename T> struct Op<OP_MUL, T, true> {
  using Acc = T;
  static __device__ __forceinline__ Acc identity() { return T(1); }
  static __device__ __forceinline__ Acc lift(T x) { return x; }
  static __device__ __forceinline__ Acc combine(Acc a, Acc b) { return a * b; }
  static __device__ __forceinline__ T finish(Acc a) { return a; }
};
// ---- floating point: max min, reading C7 (C fmax/fmin: a NaN operand is
// ignored; -0 < +0 so the result is order independent and bit exact).
// Branch-free: FMNMX already ignores a NaN operand; numerically equal operands
// (only a +-0 pair can differ in bits) combine by AND (max: +0 wins) or OR
// (min: -0 wins) of their bit patterns.
__device__ __forceinline__ float bits_and(float a, float b) { return __uint_as_float(__float_as_uint(a) & __float_as_uint(b)); }
__device__ __forceinline__ float bits_or(float a, float b) { return __uint_as_float(__float_as_uint(a) | __float_as_uint(b)); }
__device__ __forceinline__ double bits_and(double a, double b) {
  return __longlong_as_double(__double_as_longlong(a) & __double_as_longlong(b));
}
__device__ __forceinline__ double bits_or(double a, double b) {
  return __longlong_as_double(__double_as_longlong(a) | __double_as_longlong(b));
}
__device__ __forceinline__ float hw_max(float a, float b) { return fmaxf(a, b); }
__device__ __forceinline__ double hw_max(double a, double b) { return fmax(a, b); }
__device__ __forceinline__ float hw_min(float a, float b) { return fminf(a, b); }
__device__ __forceinline__ double hw_min(double a, double b) { return fmin(a, b); }
template <typename T> struct Op<OP_MAX, T, true> {
  using Acc = T;
  static __device__ __forceinline__ Acc identity() { return lowest<T>(); }
  static __device__ __forceinline__ Acc lift(T x) { return x; }
  static __device__ __forceinline__ Acc combine(Acc a, Acc b) { return a == b ? bits_and(a, b) : hw_max(a, b); }
  static __device__ __forceinline__ T finish(Acc a) { return a; }
};
template <typename T> struct Op<OP_MIN, T, true> {
  using Acc = T;
  static __device__ __forceinline__ Acc identity() { return highest<T>(); }
  static __device__ __forceinline__ Acc lift(T x) { return x; }
  static __device__ __forceinline__ Acc combine(Acc a, Acc b) { return a == b ? bits_or(a, b) : hw_min(a, b); }
  static __device__ __forceinline__ T finish(Acc a) { return a; }
};

// ---- && ||  on any type (truth = x != 0: fp NaN true, +-0 false; C8)
// The accumulator is a uint32 whose truth is "nonzero" (not 0/1): lift keeps
// the magnitude bits (fp: sign cleared, so +-0 -> 0 and NaN -> nonzero; 64-bit:
// low | high word), && combines by unsigned min (zero wins), || by OR.  One
// LOP3 / IMNMX per element in the fold instead of a compare + select + logic op.
template <typename T> __device__ __forceinline__ uint32_t truth_bits(T x) {
  if constexpr (sizeof(T) == 4) {
    uint32_t u;
    memcpy(&u, &x, 4);
    return IsFp<T>::value ? (u & 0x7fffffffu) : u;
  } else {
    unsigned long long u;
    memcpy(&u, &x, 8);
    const uint32_t lo = (uint32_t)u, hi = (uint32_t)(u >> 32);
    return lo | (IsFp<T>::value ? (hi & 0x7fffffffu) : hi);
  }
}
template <int OP, typename T> struct Logical {
  using Acc = uint32_t;
  static __device__ __forceinline__ Acc identity() { return OP == OP_LAND ? 0xffffffffu : 0u; }
  static __device__ __forceinline__ Acc lift(T x) { return truth_bits<T>(x); }
  static __device__ __forceinline__ Acc combine(Acc a, Acc b) {
    return OP == OP_LAND ? (a < b ? a : b) : (a | b);
  }
  static __device__ __forceinline__ T finish(Acc a) { return a ? T(1) : T(0); }
};
template <typename T, bool F> struct Op<OP_LAND, T, F> : Logical<OP_LAND, T> {};
template <typename T, bool F> struct Op<OP_LOR, T, F> : Logical<OP_LOR, T> {};

// ------------------------------------------------------------ a2 vector tier
// Butterfly within groups of W lanes (W a power of two <= 32); every lane of
// the warp must call it.  Full-warp groups use the hardware reductions:
//   int32 + & | ^ -> REDUX, int32 max min -> CREDUX, && || -> VOTE.
template <int OP, typename T, int W>
__device__ __forceinline__ typename Op<OP, T>::Acc butterfly(typename Op<OP, T>::Acc v) {
#pragma unroll
  for (int off = W / 2; off > 0; off >>= 1) v = Op<OP, T>::combine(v, __shfl_xor_sync(0xffffffffu, v, off));
  return v;
}

template <int OP, typename T, int W>
__device__ __forceinline__ typename Op<OP, T>::Acc group_reduce(typename Op<OP, T>::Acc v) {
  using Acc = typename Op<OP, T>::Acc;
  constexpr bool kRedux = W == 32 && sizeof(Acc) == 4 && !IsFp<Acc>::value;
  if constexpr (W == 32 && OP == OP_LAND) return __all_sync(0xffffffffu, v) ? 1u : 0u;
  else if constexpr (W == 32 && OP == OP_LOR) return __any_sync(0xffffffffu, v) ? 1u : 0u;
  else if constexpr (kRedux && OP == OP_ADD) return __reduce_add_sync(0xffffffffu, v);
  else if constexpr (kRedux && OP == OP_BAND) return __reduce_and_sync(0xffffffffu, v);
  else if constexpr (kRedux && OP == OP_BOR) return __reduce_or_sync(0xffffffffu, v);
  else if constexpr (kRedux && OP == OP_BXOR) return __reduce_xor_sync(0xffffffffu, v);
  else if constexpr (kRedux && OP == OP_MAX) return __reduce_max_sync(0xffffffffu, v);
  else if constexpr (kRedux && OP == OP_MIN) return __reduce_min_sync(0xffffffffu, v);
  else return butterfly<OP, T, W>(v);
}

// ------------------------------------------------------------ a3 worker tier
// CTA-wide combine; result valid in warp 0 (all its lanes).  smem holds
// >= 32 Acc slots.  Ends with the slots still in use: the caller must
// __syncthreads() before reusing smem.
template <int OP, typename T, int BLOCK>
__device__ __forceinline__ typename Op<OP, T>::Acc block_reduce(typename Op<OP, T>::Acc v,
                                                                typename Op<OP, T>::Acc* smem) {
  using O = Op<OP, T>;
  constexpr int NW = BLOCK / 32;
  v = group_reduce<OP, T, 32>(v);
  if constexpr (NW == 1) return v;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (lane == 0) smem[warp] = v;
  __syncthreads();
  if (warp == 0) {
    v = lane < NW ? smem[lane] : O::identity();
    v = group_reduce<OP, T, 32>(v);
  }
  return v;
}

// ------------------------------------------------------------ a4 without smem
// Workspace of grid_reduce_gmem: one Acc slot per warp of the grid and one
// zero-initialised u32 ticket (self-resetting); caller-owned device memory.
template <typename Acc> struct GmemWorkspace {
  Acc* warp_partials;  // >= total warps of the launch
  unsigned* ticket;    // 1, zero before the first launch
};

// Gang tier with NO shared memory: every warp (all lanes must call) combines
// its lanes with shuffles, lane 0 stores the warp partial in global memory,
// fences and takes the ticket; the LAST warp of the grid folds all warp
// partials in warp order (deterministic for a fixed launch) and writes
// out = init (+) R (init = *out if init_from_out, else the identity).
// Returns true in the lanes of the warp that wrote *out.
template <int OP, typename T>
__device__ __forceinline__ bool grid_reduce_gmem(typename Op<OP, T>::Acc v, GmemWorkspace<typename Op<OP, T>::Acc> ws,
                                                 T* out, bool init_from_out = false) {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  const unsigned lane = threadIdx.x & 31u;
  const unsigned wpb = (blockDim.x * blockDim.y * blockDim.z + 31u) / 32u;
  const unsigned tflat = threadIdx.x + blockDim.x * (threadIdx.y + blockDim.y * threadIdx.z);
  const unsigned bflat = blockIdx.x + gridDim.x * (blockIdx.y + gridDim.y * blockIdx.z);
  const unsigned long long gw = (unsigned long long)bflat * wpb + tflat / 32u;
  const unsigned long long nw = (unsigned long long)gridDim.x * gridDim.y * gridDim.z * wpb;
  v = group_reduce<OP, T, 32>(v);
  unsigned last = 0;
  if (lane == 0) {
    ws.warp_partials[gw] = v;
    __threadfence();
    last = (atomicAdd(ws.ticket, 1u) == (unsigned)(nw - 1ull));
  }
  last = __shfl_sync(0xffffffffu, last, 0);
  if (!last) return false;
  __threadfence();
  Acc w = O::identity();
  for (unsigned long long i = lane; i < nw; i += 32ull) w = O::combine(w, __ldcg(ws.warp_partials + i));
  w = group_reduce<OP, T, 32>(w);
  if (lane == 0) {
    const Acc init = init_from_out ? O::lift(*out) : O::identity();
    *out = O::finish(O::combine(init, w));
    *ws.ticket = 0u;
  }
  return true;
}

}  // namespace xr
