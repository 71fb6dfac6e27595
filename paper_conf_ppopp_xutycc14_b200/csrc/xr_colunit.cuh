// xr_colunit.cuh -- one CTA-wide column unit (RK / KRK shapes) over a generic
// element "lifter" X, for the launches that fuse more than one input or more
// than one variable into one pass: the transform-reduce (two inputs, PAPER.md
// Fig 13(b)/(c)) and the multi-variable reduction (PAPER.md
// 3.3 @31605-32570).  Same decomposition and tiers as the
// library's col_kernel (xr_kernels.cuh): lanes own VEC contiguous kept
// columns (a 32*VEC-column tile), the CTA's warps stride the reduced rows of a
// row chunk (a1), the worker tier folds the per-warp column partials in
// shared memory in fixed warp order (a3, @21991-24615), and the gang tier is
// a per-tile ticket whose last CTA folds the S chunk partials (a4, replacing
// the paper's partial buffer + second launch, @24887-25280).
//
// X provides: Acc, Out, identity(), combine(a, b), lift(T x, T y) (y is
// ignored when NIN == 1), lift_out(Out) (the prior output as an init, a5) and
// finish(Acc).
#pragma once
#include "xr_internal.h"
#include "xr_ops.cuh"

namespace xr {

// Op<OP, T> as a one-input lifter (the multi-variable launch).
template <int OP, typename T>
struct OpLift {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  using Out = T;
  static __device__ __forceinline__ Acc identity() { return O::identity(); }
  static __device__ __forceinline__ Acc combine(Acc a, Acc b) { return O::combine(a, b); }
  static __device__ __forceinline__ Acc lift(T x, T) { return O::lift(x); }
  static __device__ __forceinline__ Acc lift_out(Out v) { return O::lift(v); }
  static __device__ __forceinline__ Out finish(Acc a) { return O::finish(a); }
};

__device__ __forceinline__ int64_t cu_split(int64_t n, int64_t parts, int64_t i) {
  const int64_t q = n / parts, r = n % parts;
  return i * q + (i < r ? i : r);
}

// Shared memory a unit needs: [kBlock/32 warps][32*VEC columns] accumulators.
template <class X, int VEC>
constexpr int col_unit_smem() {
  return (kBlock / 32) * 32 * VEC * (int)sizeof(typename X::Acc);
}

// Unit u of the column decomposition a (u in [0, a.units)): in0 / in1 are the
// inputs (in1 unused when NIN == 1); a.out / a.partials / a.tickets as in
// col_kernel.  sm: col_unit_smem<X, VEC>() bytes.  Every thread of the CTA
// calls it; it ends with a barrier, so sm can be reused by the next unit.
template <class X, typename T, int NIN, int VEC, int U>
__device__ __forceinline__ void col_unit(const ColArgs& a, const T* __restrict__ in0, const T* __restrict__ in1,
                                         int64_t u, void* sm_raw, int* s_last) {
  using Acc = typename X::Acc;
  using Out = typename X::Out;
  constexpr int NW = kBlock / 32;
  constexpr int TW = 32 * VEC;
  Acc (*sm)[TW] = reinterpret_cast<Acc (*)[TW]>(sm_raw);
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, t = threadIdx.x;
  Out* out = static_cast<Out*>(a.out);
  Acc* partials = static_cast<Acc*>(a.partials);
  const int64_t per_b = a.tiles * a.S;
  const int64_t b = u / per_b, rem = u - b * per_b;
  const int64_t tile = rem / a.S, s = rem - tile * a.S;
  const int64_t col = tile * TW + (int64_t)lane * VEC;
  const int64_t r0 = cu_split(a.R, a.S, s), r1 = cu_split(a.R, a.S, s + 1);
  Acc acc[U][VEC];
#pragma unroll
  for (int k = 0; k < U; ++k)
#pragma unroll
    for (int q = 0; q < VEC; ++q) acc[k][q] = X::identity();
  if (col < a.K) {  // VEC > 1 only when K % VEC == 0: the lane owns VEC whole columns
    const int64_t off = b * a.R * a.K + col;
    int64_t r = r0 + warp;
    if constexpr (VEC > 1) {
      for (; r + (int64_t)(U - 1) * NW < r1; r += (int64_t)U * NW) {
        U128 x[U], y[U];
#pragma unroll
        for (int k = 0; k < U; ++k) {
          x[k] = ld_stream(in0 + off + (r + (int64_t)k * NW) * a.K);
          if constexpr (NIN == 2) y[k] = ld_stream(in1 + off + (r + (int64_t)k * NW) * a.K);
        }
#pragma unroll
        for (int k = 0; k < U; ++k)
#pragma unroll
          for (int q = 0; q < VEC; ++q)
            acc[k][q] = X::combine(acc[k][q], X::lift(unpack<T>(x[k], q), NIN == 2 ? unpack<T>(y[k], q) : T(0)));
      }
      for (; r < r1; r += NW) {
        const U128 x = ld_stream(in0 + off + r * a.K);
        U128 y{};
        if constexpr (NIN == 2) y = ld_stream(in1 + off + r * a.K);
#pragma unroll
        for (int q = 0; q < VEC; ++q)
          acc[0][q] = X::combine(acc[0][q], X::lift(unpack<T>(x, q), NIN == 2 ? unpack<T>(y, q) : T(0)));
      }
    } else {
      for (; r + (int64_t)(U - 1) * NW < r1; r += (int64_t)U * NW) {
        T x[U], y[U];
#pragma unroll
        for (int k = 0; k < U; ++k) {
          x[k] = ld_scalar(in0 + off + (r + (int64_t)k * NW) * a.K);
          y[k] = NIN == 2 ? ld_scalar(in1 + off + (r + (int64_t)k * NW) * a.K) : T(0);
        }
#pragma unroll
        for (int k = 0; k < U; ++k) acc[k][0] = X::combine(acc[k][0], X::lift(x[k], y[k]));
      }
      for (; r < r1; r += NW)
        acc[0][0] = X::combine(acc[0][0], X::lift(ld_scalar(in0 + off + r * a.K),
                                                  NIN == 2 ? ld_scalar(in1 + off + r * a.K) : T(0)));
    }
  }
#pragma unroll
  for (int k = 1; k < U; ++k)
#pragma unroll
    for (int q = 0; q < VEC; ++q) acc[0][q] = X::combine(acc[0][q], acc[k][q]);
#pragma unroll
  for (int q = 0; q < VEC; ++q) sm[warp][lane * VEC + q] = acc[0][q];
  __syncthreads();
  // a3: worker tier, fixed warp order per column
  Acc v = X::identity();
  if (t < TW) {
#pragma unroll
    for (int w = 0; w < NW; ++w) v = X::combine(v, sm[w][t]);
  }
  const int64_t oc = tile * TW + t;
  if (a.S == 1) {
    if (t < TW && oc < a.K) {
      const int64_t o = b * a.K + oc;
      const Acc init = a.init_from_out ? X::lift_out(out[o]) : X::identity();
      out[o] = X::finish(X::combine(init, v));
    }
  } else {  // a4: gang tier per column tile
    Acc* P = partials + (b * a.tiles + tile) * a.S * TW;
    if (t < TW) P[s * TW + t] = v;
    __syncthreads();  // the CTA's partial stores happen-before thread 0's fence (cumulative)
    if (t == 0) *s_last = (ticket_add(&a.tickets[b * a.tiles + tile]) == (unsigned)(a.S - 1));
    __syncthreads();
    if (*s_last) {
      __threadfence();
      Acc w2[VEC];
#pragma unroll
      for (int q = 0; q < VEC; ++q) w2[q] = X::identity();
      for (int64_t si = warp; si < a.S; si += NW)
#pragma unroll
        for (int q = 0; q < VEC; ++q) w2[q] = X::combine(w2[q], ld_partial(P + si * TW + lane * VEC + q));
#pragma unroll
      for (int q = 0; q < VEC; ++q) sm[warp][lane * VEC + q] = w2[q];
      __syncthreads();
      if (t < TW && oc < a.K) {
        Acc z = X::identity();
#pragma unroll
        for (int w = 0; w < NW; ++w) z = X::combine(z, sm[w][t]);
        const int64_t o = b * a.K + oc;
        const Acc init = a.init_from_out ? X::lift_out(out[o]) : X::identity();
        out[o] = X::finish(X::combine(init, z));
      }
      if (t == 0) a.tickets[b * a.tiles + tile] = 0u;
    }
  }
  __syncthreads();
}

}  // namespace xr
