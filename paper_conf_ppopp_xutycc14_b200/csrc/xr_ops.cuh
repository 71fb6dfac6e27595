// xr_ops.cuh -- operator traits and the three combine tiers (sm_100a).
//
// Tier mapping:
//   a1 private partials : identity-initialised register accumulators, the
//                         paper's "each vector thread first creates a private
//                         variable and does the partial reduction itself"
//                         (PAPER.md @19558-19752, 3.1.1; Fig 5 i_sum_priv).
//   a2 vector tier      : intra-warp combine with REDUX / VOTE / SHFL instead
//                         of the shared-memory interleaved log-step of Fig 7
//                         (@19365-21328).
//   a3 worker tier      : cross-warp combine through <=32 shared-memory slots
//                         and one barrier, cf. Fig 8(c) "the first vector thread
//                         of each worker stores the partial ... into the shared
//                         memory" (@23603-24615).
//   a4 gang tier        : per-CTA partial + last-CTA-done ticket (xr_kernels.cu)
//                         instead of "another kernel ... launched" (@24887-25280).
// All operators are associative and commutative, so any combine order is
// licensed (@15024-15239, 3); fixed grids make the order deterministic.
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
//   && ||          : uint32 truth value (C8)
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
template <int OP, typename T> struct Logical {
  using Acc = uint32_t;
  static __device__ __forceinline__ Acc identity() { return OP == OP_LAND ? 1u : 0u; }
  static __device__ __forceinline__ Acc lift(T x) { return x != T(0) ? 1u : 0u; }
  static __device__ __forceinline__ Acc combine(Acc a, Acc b) {
    return OP == OP_LAND ? (a & b) : (a | b);
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

// ------------------------------------------------------------ memory helpers
// 16-byte streaming load: read once, no L1 allocation (non-coherent path:
// the input is read-only for the kernel's lifetime).
struct alignas(16) U128 { uint32_t w[4]; };

__device__ __forceinline__ U128 ld_stream(const void* p) {
  U128 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.w[0]), "=r"(r.w[1]), "=r"(r.w[2]), "=r"(r.w[3])
               : "l"(p));
  return r;
}

template <typename T> __device__ __forceinline__ T ld_scalar(const T* p) { return __ldg(p); }

// L2-coherent load of a partial written by another CTA of the same grid.
template <typename A> __device__ __forceinline__ A ld_partial(const A* p) { return __ldcg(p); }

template <typename T> __device__ __forceinline__ T unpack(const U128& u, int q) {
  static_assert(sizeof(T) == 4 || sizeof(T) == 8, "dtype");
  if constexpr (sizeof(T) == 4) {
    if constexpr (IsFp<T>::value) return __uint_as_float(u.w[q]);
    else return static_cast<T>(u.w[q]);
  } else {
    const unsigned long long b =
        (unsigned long long)u.w[2 * q] | ((unsigned long long)u.w[2 * q + 1] << 32);
    if constexpr (IsFp<T>::value) return __longlong_as_double((long long)b);
    else return static_cast<T>(b);
  }
}

}  // namespace xr

namespace xr {
// ------------------------------------------------------------ bulk async copy
// cp.async.bulk (the TMA engine's 1-D copy, SASS UBLKCP) global -> shared,
// completing on an mbarrier with a transaction byte count.
__device__ __forceinline__ unsigned smem_addr(const void* p) {
  return static_cast<unsigned>(__cvta_generic_to_shared(p));
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, unsigned count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_addr(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void fence_mbar_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, unsigned bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_addr(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, unsigned bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_addr(dst)),
      "l"(src), "r"(bytes), "r"(smem_addr(bar))
      : "memory");
}
// TMA tensor load of one box (3-D map: {column, row, batch}) into shared memory.
__device__ __forceinline__ void tma_load_3d(void* dst, const void* tmap, int c0, int c1, int c2, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4}], [%5];" ::
          "r"(smem_addr(dst)),
      "l"(reinterpret_cast<uint64_t>(tmap)), "r"(c0), "r"(c1), "r"(c2), "r"(smem_addr(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, unsigned parity) {
  asm volatile(
      "{\n\t.reg .pred p;\n"
      "XR_WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n\t"
      "@!p bra XR_WAIT_%=;\n}" ::"r"(smem_addr(bar)),
      "r"(parity)
      : "memory");
}
}  // namespace xr

namespace xr {
// ------------------------------------------------------------ warp specialisation
// Producer warp + kConsWarps consumer warps: the consumers synchronise among
// themselves with named barrier 1 (never with the producer), and release a
// stage by one arrival per consumer warp on its "empty" mbarrier.
constexpr int kConsWarps = 8;
constexpr int kConsThreads = 32 * kConsWarps;
constexpr int kWsBlock = kConsThreads + 32;  // + the producer warp

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_addr(bar)) : "memory");
}
__device__ __forceinline__ void cons_sync() {
  asm volatile("bar.sync 1, %0;" ::"n"(kConsThreads) : "memory");
}
// Consumer-wide combine (a2 + a3); result valid in consumer warp 0.  The
// caller must cons_sync() before reusing smem.
template <int OP, typename T>
__device__ __forceinline__ typename Op<OP, T>::Acc cons_reduce(typename Op<OP, T>::Acc v,
                                                               typename Op<OP, T>::Acc* smem, int cw,
                                                               int lane) {
  v = group_reduce<OP, T, 32>(v);
  if (lane == 0) smem[cw] = v;
  cons_sync();
  if (cw == 0) {
    v = lane < kConsWarps ? smem[lane] : Op<OP, T>::identity();
    v = group_reduce<OP, T, 32>(v);
  }
  return v;
}
}  // namespace xr
