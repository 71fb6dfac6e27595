// xr_kernels.cuh -- the reduction kernels (sm_100a), one family per canonical
// shape (xr_plan.cpp).  Every launch is single pass: per-CTA (or per-warp)
// partials are combined by the LAST unit to finish, found with an atomic
// ticket after a __threadfence() -- the gang tier of SURVEY.md 8(a) a4, which
// replaces the paper's "temporary buffer (partial in Figure 5(c)) ... then
// another kernel ... is launched" (PAPER.md @24887-25280, 3.1.3) and the RMP
// global buffer + second kernel (@29217-29414, @31388-31587).
#pragma once
#include <cuda.h>

#include <algorithm>
#include <cstdlib>

#include "xr_internal.h"
#include "xr_ops.cuh"

namespace xr {

// [lo, hi) of part `i` when n items are split in `parts` near-equal parts.
__device__ __forceinline__ int64_t split_lo(int64_t n, int64_t parts, int64_t i) {
  const int64_t q = n / parts, r = n % parts;
  return i * q + (i < r ? i : r);
}
// Same, rounded down to a multiple of `v` (except the end, which is n).
__device__ __forceinline__ int64_t split_lo_vec(int64_t n, int64_t parts, int64_t i, int v) {
  if (i >= parts) return n;
  return (split_lo(n, parts, i) / v) * v;
}

// Rows [r0, r1) of split s when R rows are split in S parts at whole boxes of
// BR rows (no TMA box straddles two units, so no row is fetched twice).
__device__ __forceinline__ void box_rows(int64_t R, int64_t S, int64_t s, int BR, int64_t* r0, int64_t* r1) {
  const int64_t nb = (R + BR - 1) / BR;
  *r0 = min(split_lo(nb, S, s) * BR, R);
  *r1 = min(split_lo(nb, S, s + 1) * BR, R);
}

// ------------------------------------------------------------- a1 (rows)
// Fold row[0..n) into the lane's private accumulators: a scalar head up to the
// first 16-B boundary, 16-B vectors strided by the group width W with U loads
// in flight, then a scalar tail.  Works for any dtype-aligned row start (the
// paper's arbitrary iteration spaces, @33355-34930; reading C19).
template <int OP, typename T, int W, int U>
__device__ __forceinline__ void fold_row(const T* __restrict__ row, int64_t n, int lane,
                                         typename Op<OP, T>::Acc (&acc)[U][16 / sizeof(T)]) {
  using O = Op<OP, T>;
  constexpr int VEC = 16 / sizeof(T);
  int64_t head = (int64_t)((16u - ((uint32_t)(uintptr_t)row & 15u)) & 15u) / (int64_t)sizeof(T);
  if (head > n) head = n;
  if (lane < head) acc[0][0] = O::combine(acc[0][0], O::lift(ld_scalar(row + lane)));
  row += head;
  n -= head;
  const int64_t nv = n / VEC;
  const U128* __restrict__ vp = reinterpret_cast<const U128*>(row);
  int64_t v = lane;
// XR_FOLD_PIPELINE=1: software-pipelined variant (A/B only; more registers,
// measured no better than the plain loop under __launch_bounds__(256, 4))
#ifndef XR_FOLD_PIPELINE
#define XR_FOLD_PIPELINE 0
#endif
#if XR_FOLD_PIPELINE == 0
  for (; v + (int64_t)(U - 1) * W < nv; v += (int64_t)U * W) {
    U128 x[U];
#pragma unroll
    for (int k = 0; k < U; ++k) x[k] = ld_stream(vp + v + (int64_t)k * W);
#pragma unroll
    for (int k = 0; k < U; ++k)
#pragma unroll
      for (int q = 0; q < VEC; ++q) acc[k][q] = O::combine(acc[k][q], O::lift(unpack<T>(x[k], q)));
  }
#else
  if (v + (int64_t)(U - 1) * W < nv) {
    // software-pipelined: the U loads of round n+1 are issued before round n
    // is folded, so they have no use inside the iteration and ptxas keeps
    // them in one batch (it sank unpipelined loads next to their uses,
    // leaving 2 of 4 in flight: fp64 && || rows at 0.63 of peak, r01)
    U128 x[U];
#pragma unroll
    for (int k = 0; k < U; ++k) x[k] = ld_stream(vp + v + (int64_t)k * W);
    v += (int64_t)U * W;
    for (; v + (int64_t)(U - 1) * W < nv; v += (int64_t)U * W) {
      U128 y[U];
#pragma unroll
      for (int k = 0; k < U; ++k) y[k] = ld_stream(vp + v + (int64_t)k * W);
#pragma unroll
      for (int k = 0; k < U; ++k)
#pragma unroll
        for (int q = 0; q < VEC; ++q) acc[k][q] = O::combine(acc[k][q], O::lift(unpack<T>(x[k], q)));
#pragma unroll
      for (int k = 0; k < U; ++k) x[k] = y[k];
    }
#pragma unroll
    for (int k = 0; k < U; ++k)
#pragma unroll
      for (int q = 0; q < VEC; ++q) acc[k][q] = O::combine(acc[k][q], O::lift(unpack<T>(x[k], q)));
  }
#endif
  for (; v < nv; v += W) {
    const U128 x = ld_stream(vp + v);
#pragma unroll
    for (int q = 0; q < VEC; ++q) acc[0][q] = O::combine(acc[0][q], O::lift(unpack<T>(x, q)));
  }
  const int64_t tail = n - nv * VEC;
  if (lane < tail) acc[1 % U][0] = O::combine(acc[1 % U][0], O::lift(ld_scalar(row + nv * VEC + lane)));
}

// Combine the U x VEC private accumulators in a fixed pairwise order.
template <int OP, typename T, int U, int VEC>
__device__ __forceinline__ typename Op<OP, T>::Acc fold_acc(typename Op<OP, T>::Acc (&acc)[U][VEC]) {
  using O = Op<OP, T>;
#pragma unroll
  for (int k = 1; k < U; ++k)
#pragma unroll
    for (int q = 0; q < VEC; ++q) acc[0][q] = O::combine(acc[0][q], acc[k][q]);
#pragma unroll
  for (int w = VEC / 2; w > 0; w >>= 1)
#pragma unroll
    for (int q = 0; q < w; ++q) acc[0][q] = O::combine(acc[0][q], acc[0][q + w]);
  return acc[0][0];
}

// This lane's partial over work unit u of a seg launch.
template <int OP, typename T, int W, int U>
__device__ __forceinline__ typename Op<OP, T>::Acc seg_unit(const SegArgs& a, int64_t u, int lane,
                                                            int64_t* o_out) {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  constexpr int VEC = 16 / sizeof(T);
  int64_t o, r0, r1, c0, c1;
  if (a.Sr == 1 && a.Sc == 1) {  // unsplit: no 64-bit divisions on the per-row path
    o = u; r0 = 0; r1 = a.C; c0 = 0; c1 = a.L;
  } else {
    const int64_t S = a.Sr * a.Sc;
    o = u / S;
    const int64_t s = u - o * S;
    const int64_t sr = s / a.Sc, sc = s - sr * a.Sc;
    r0 = split_lo(a.C, a.Sr, sr); r1 = split_lo(a.C, a.Sr, sr + 1);
    c0 = split_lo_vec(a.L, a.Sc, sc, VEC); c1 = split_lo_vec(a.L, a.Sc, sc + 1, VEC);
  }
  Acc acc[U][VEC];
#pragma unroll
  for (int k = 0; k < U; ++k)
#pragma unroll
    for (int q = 0; q < VEC; ++q) acc[k][q] = O::identity();
  const T* __restrict__ base = static_cast<const T*>(a.in) + o * a.oStride + c0;
  for (int64_t r = r0; r < r1; ++r) fold_row<OP, T, W, U>(base + r * a.rowStride, c1 - c0, lane, acc);
  *o_out = o;
  return fold_acc<OP, T, U, VEC>(acc);
}

// Fused exchange (one thread): publish `mine` to every rank's mailbox, wait for
// all ranks (bounded by timeout_ns of %globaltimer), then out[0] = combine of
// the nranks values in rank order -- identical bits on every rank.  `mine`
// already carries this rank's share of the initial value (rank 0 only,
// xr_shard_plan).  If a peer does not arrive in time, out is left UNCHANGED
// and the host-mapped status word is set (the host reports XR_ERR_NCCL on the
// next call and through xr_comm_query); a stale combine is never written.
template <int OP, typename T>
__device__ __noinline__ void peer_exchange(const ExchArgs& ex, T* out, T mine) {
  const ExchArgs* x = &ex;
  using O = Op<OP, T>;
  unsigned long long bits = 0ull;
  memcpy(&bits, &mine, sizeof(T));
  const int par = (int)(x->epoch & 1ull);
  for (int p = 0; p < x->nranks; ++p) x->peers[p][par * kMaxRanks + x->rank] = bits;  // NVLink stores
  // each flag store is a release at system scope: it orders this thread's
  // slot stores above before the flag becomes visible to the peer
  for (int p = 0; p < x->nranks; ++p) {
    unsigned long long* f = x->peers[p] + 2 * kMaxRanks + x->rank;
    asm volatile("st.release.sys.global.u64 [%0], %1;" ::"l"(f), "l"(x->epoch) : "memory");
  }
  const unsigned long long t0 = globaltimer_ns();
  typename O::Acc acc = O::identity();
  for (int q = 0; q < x->nranks; ++q) {
    const unsigned long long* f = x->mine + 2 * kMaxRanks + q;
    unsigned long long e = 0ull;
    while (true) {
      asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(e) : "l"(f) : "memory");
      if (e >= x->epoch) break;
      if (globaltimer_ns() - t0 > x->timeout_ns) {  // a peer never arrived: report, do not hang
        *reinterpret_cast<volatile int*>(x->status) = 1;
        __threadfence_system();
        return;
      }
      __nanosleep(64);
    }
    unsigned long long v;
    asm volatile("ld.relaxed.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(x->mine + par * kMaxRanks + q) : "memory");
    T tv;
    memcpy(&tv, &v, sizeof(T));
    acc = O::combine(acc, O::lift(tv));
  }
  out[0] = O::finish(acc);
}

// a5: out[o] = init (+) R, init = identity or the prior out[o] (@21488-21990).
template <int OP, typename T>
__device__ __forceinline__ T merge_init(typename Op<OP, T>::Acc v, const T* out, int64_t o,
                                        int init_from_out) {
  using O = Op<OP, T>;
  const typename O::Acc init = init_from_out ? O::lift(out[o]) : O::identity();
  return O::finish(O::combine(init, v));
}

// Fold p[start], p[start+stride], ... (< n) with 8 independent L2 loads in
// flight per round (the last-CTA combine is latency bound, not bandwidth bound).
template <int OP, typename T>
__device__ __forceinline__ typename Op<OP, T>::Acc fold_partials(const typename Op<OP, T>::Acc* p, int64_t n,
                                                                 int64_t start, int64_t stride) {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  Acc w = O::identity();
  int64_t i = start;
  for (; i + 7 * stride < n; i += 8 * stride) {
    Acc y[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) y[k] = ld_partial(p + i + k * stride);
#pragma unroll
    for (int k = 0; k < 8; ++k) w = O::combine(w, y[k]);
  }
  for (; i < n; i += stride) w = O::combine(w, ld_partial(p + i));
  return w;
}

// Fold a CONTIGUOUS 16-B aligned partial array p[0..n) with 16-B loads (4 or 2
// accumulators each), 8 in flight per thread: the single-output "whole" mode
// folds thousands of unit partials after every other CTA has finished, so
// this tail is latency bound (r01: 9472 partials in 5 rounds of 8 scalar
// loads per thread -> 2 rounds of 16-B loads).  Fixed order per thread.
template <int OP, typename T>
__device__ __forceinline__ typename Op<OP, T>::Acc fold_partials_vec(const typename Op<OP, T>::Acc* p, int64_t n,
                                                                     int t, int nt) {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  constexpr int PV = 16 / sizeof(Acc);
  const int64_t nv = n / PV;
  Acc w = O::identity();
  int64_t i = t;
  for (; i + 7 * (int64_t)nt < nv; i += 8 * (int64_t)nt) {
    U128 y[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) y[k] = ld_partial16(p + (i + (int64_t)k * nt) * PV);
#pragma unroll
    for (int k = 0; k < 8; ++k)
#pragma unroll
      for (int q = 0; q < PV; ++q) w = O::combine(w, acc_at<Acc>(y[k], q));
  }
  for (; i < nv; i += nt) {
    const U128 y = ld_partial16(p + i * PV);
#pragma unroll
    for (int q = 0; q < PV; ++q) w = O::combine(w, acc_at<Acc>(y, q));
  }
  for (int64_t e = nv * PV + t; e < n; e += nt) w = O::combine(w, ld_partial(p + e));
  return w;
}

// ------------------------------------------------------------- seg kernel
// Groups of W lanes (8 or 32: inside a warp; W == BLOCK: the whole CTA) each
// reduce work units; a unit is (output o, split s).  Splits (S > 1) only
// occur with W >= 32 (plan), so a ticket is always taken by a whole warp/CTA.
template <int OP, typename T, int W, int BLOCK, int U>
// Minimum resident CTAs in the register kernels' launch bounds (<= 64
// registers).  It also steers ptxas's scheduling: without it ptxas sank the
// unrolled 16-B loads of fold_row next to their uses in some instantiations
// (2 of 4 loads in flight; fp64 && || rows at 0.63 of peak, the paper's
// 2^20 x 2 x 32 gang case at 64 us instead of 50 us).  r01 A/B, and
// tests/test_sass.py keeps every fold loop at >= 4 loads in flight.
#ifndef XR_SEG_MINB
#define XR_SEG_MINB 4
#endif
__global__ void __launch_bounds__(BLOCK, XR_SEG_MINB) seg_kernel(const __grid_constant__ SegArgs a) {
  pdl_wait();  // no global access above this line
  pdl_trigger();
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  __shared__ Acc smem[32];
  __shared__ int s_last;
  T* out = static_cast<T*>(a.out);
  Acc* partials = static_cast<Acc*>(a.partials);
  const int64_t S = a.Sr * a.Sc;

  if constexpr (W == BLOCK) {
    __shared__ long long s_unit[2];
    // one unit per CTA (small, latency-bound inputs): static assignment, no
    // claim round trip at the start and no exit counter at the end
    // a.seg_static (A/B): every CTA takes units blockIdx.x + i * gridDim.x,
    // no claims at all
    const bool one_each = a.units <= (int64_t)gridDim.x;
    const bool stat = one_each || a.seg_static;
    if (threadIdx.x == 0) s_unit[0] = stat ? (long long)blockIdx.x : claim_first(a.sched);
    __syncthreads();
    long long u = s_unit[0];
    int par = 1;
    while (u < a.units) {
      if (threadIdx.x == 0) s_unit[par] = stat ? u + (long long)gridDim.x : claim_next(a.sched);  // next, in flight
      int64_t o;
      Acc v = seg_unit<OP, T, W, U>(a, u, threadIdx.x, &o);
      v = block_reduce<OP, T, BLOCK>(v, smem);  // a2 + a3
      if (S == 1) {
        if (threadIdx.x == 0) {
          const T r = merge_init<OP, T>(v, out, o, a.init_from_out);
          if (a.use_exch) peer_exchange<OP, T>(a.exch, out, r);
          else out[o] = r;
        }
      } else if (PackedAdd<OP, T>::value && a.packed) {  // a4 in one atomic (32-bit int '+')
        uint32_t sum;
        if (threadIdx.x == 0 &&
            packed_add_arrive(reinterpret_cast<unsigned long long*>(a.tickets) + o, (uint32_t)v, S, &sum)) {
          const T r = merge_init<OP, T>((Acc)sum, out, o, a.init_from_out);
          if (a.use_exch) peer_exchange<OP, T>(a.exch, out, r);
          else out[o] = r;
        }
      } else {  // a4: gang tier, last CTA of output o combines its S partials
        if (threadIdx.x == 0) {
          partials[u] = v;
          const unsigned t = ticket_add(&a.tickets[o]);
          s_last = (t == (unsigned)(S - 1));
        }
        __syncthreads();
        if (s_last) {
          __threadfence();
          Acc w = fold_partials<OP, T>(partials + o * S, S, threadIdx.x, BLOCK);
          w = block_reduce<OP, T, BLOCK>(w, smem);
          if (threadIdx.x == 0) {
            const T r = merge_init<OP, T>(w, out, o, a.init_from_out);
            a.tickets[o] = 0u;  // self-resetting for the next launch
            if (a.use_exch) peer_exchange<OP, T>(a.exch, out, r);
            else out[o] = r;
          }
        }
      }
      __syncthreads();
      u = s_unit[par];
      par ^= 1;
    }
    if (!stat) sched_exit(a.sched);
  } else {
    static_assert(W <= 32 && (32 % W) == 0, "sub-warp group");
    const int lane = threadIdx.x & (W - 1);
    const int64_t gid = ((int64_t)blockIdx.x * BLOCK + threadIdx.x) / W;
    const int64_t gid0 = gid - (int64_t)((threadIdx.x & 31) / W);  // first group of my warp
    const int64_t G = (int64_t)gridDim.x * (BLOCK / W);
    // warp-uniform trip count so every lane reaches the shuffles together
    for (int64_t b = gid0; b < a.units; b += G) {
      const int64_t u = b + (gid - gid0);
      const bool active = u < a.units;
      int64_t o = 0;
      Acc v = active ? seg_unit<OP, T, W, U>(a, u, lane, &o) : O::identity();
      v = group_reduce<OP, T, W>(v);
      if (S == 1) {
        if (active && lane == 0) out[o] = merge_init<OP, T>(v, out, o, a.init_from_out);
      } else if (PackedAdd<OP, T>::value && a.packed) {  // a4 in one atomic (32-bit int '+')
        uint32_t sum;
        if (active && lane == 0 &&
            packed_add_arrive(reinterpret_cast<unsigned long long*>(a.tickets) + o, (uint32_t)v, S, &sum))
          out[o] = merge_init<OP, T>((Acc)sum, out, o, a.init_from_out);
      } else {  // W == 32 here: the warp is one group, `active` is warp-uniform
        int last = 0;
        if (lane == 0) {
          partials[u] = v;
          const unsigned t = ticket_add(&a.tickets[o]);
          last = (t == (unsigned)(S - 1));
        }
        last = __shfl_sync(0xffffffffu, last, 0);
        if (last) {
          __threadfence();
          Acc w = fold_partials<OP, T>(partials + o * S, S, lane, 32);
          w = group_reduce<OP, T, 32>(w);
          if (lane == 0) {
            out[o] = merge_init<OP, T>(w, out, o, a.init_from_out);
            a.tickets[o] = 0u;
          }
        }
      }
    }
  }
}

// ------------------------------------------------------------- stream kernel
// The warp-specialised ring kernels (stream, rows, rkr, coltma) run 3 CTAs per
// SM (64 KiB ring each); declaring that residency lets ptxas keep every
// shared-memory load of a stage in flight instead of reusing one register
// quadruple per load (r01 SASS: serialized LDS.128 chains without it).
#ifndef XR_WS_MINB
#define XR_WS_MINB 3
#endif
// R and long-row KR shapes (C == 1): each unit is one contiguous range; RKR
// with 16-B aligned rows (C > 1): each unit is a run of whole rows of one
// output at the row stride, and the stages are filled from the rows'
// concatenation (a fold does not care where a row ends).  The unit's
// 16-B-aligned body is streamed into a ring of NS shared-memory stages by the
// TMA bulk-copy engine (cp.async.bulk, completion on an mbarrier with a byte
// count); thread 0 is the producer and keeps NS stages (NS*STAGE bytes) in
// flight ACROSS unit boundaries, so memory-level parallelism no longer depends
// on registers or per-element ALU cost.  All threads fold the stage from
// shared memory (a1), then the warp / CTA / last-CTA tiers run as in seg.
struct StreamGeom {
  int64_t o;
  int64_t head, nbody, tail;  // elements
  const void* row;
};

template <typename T>
__device__ __forceinline__ StreamGeom stream_geom(const SegArgs& a, long long u) {
  constexpr int VEC = 16 / sizeof(T);
  StreamGeom g;
  if (a.C > 1) {  // RKR: whole 16-B aligned rows r0..r1-1 of output o (plan), no head / tail
    const int64_t S = a.Sr;
    int64_t s;
    if (a.smaj) {  // split-major ids: concurrent units cover every output of one row range
      s = u / a.O;
      g.o = u - s * a.O;
    } else {
      g.o = u / S;
      s = u - g.o * S;
    }
    const int64_t r0 = split_lo(a.C, S, s), r1 = split_lo(a.C, S, s + 1);
    g.row = static_cast<const T*>(a.in) + g.o * a.oStride + r0 * a.rowStride;
    g.head = 0;
    g.tail = 0;
    g.nbody = (r1 - r0) * a.L;
    return g;
  }
  int64_t c0, c1;
  if (a.gd.nph > 0) {  // guided units of the whole-array shape (O == 1)
    int k = 0;
    while (k + 1 < a.gd.nph && u >= a.gd.u0[k + 1]) ++k;
    g.o = 0;
    c0 = a.gd.c0[k] + (u - a.gd.u0[k]) * a.gd.len[k];
    c1 = min(c0 + a.gd.len[k], a.gd.c0[k + 1]);
  } else {
    const int64_t S = a.Sc;
    g.o = u / S;
    const int64_t s = u - g.o * S;
    c0 = split_lo_vec(a.L, S, s, VEC);
    c1 = split_lo_vec(a.L, S, s + 1, VEC);
  }
  const T* row = static_cast<const T*>(a.in) + g.o * a.oStride + c0;
  const int64_t n = c1 - c0;
  int64_t head = (int64_t)((16u - ((uint32_t)(uintptr_t)row & 15u)) & 15u) / (int64_t)sizeof(T);
  if (head > n) head = n;
  g.head = head;
  g.nbody = ((n - head) / VEC) * VEC;
  g.tail = n - head - g.nbody;
  g.row = row;
  return g;
}

template <int OP, typename T, int NS, int STAGE>
__global__ void __launch_bounds__(kWsEpiBlock, XR_WS_MINB) stream_kernel(const __grid_constant__ SegArgs a) {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  constexpr int VEC = 16 / sizeof(T);
  constexpr int PER = STAGE / (16 * kConsThreads);  // 16-B vectors per consumer thread per stage
  constexpr int RING = 8;                           // published unit ids
  static_assert(PER >= 1 && STAGE % (16 * kConsThreads) == 0, "stage geometry");
  extern __shared__ __align__(1024) unsigned char stage_mem[];  // NS * STAGE
  __shared__ __align__(8) uint64_t full[NS];
  __shared__ __align__(8) uint64_t empty[NS];
  __shared__ long long s_units[RING];
  __shared__ Acc smem[32];
  __shared__ int s_last;
  // per-output gang tier handed to the epilogue warp: a mailbox of RING unit
  // results (unit id, CTA value), full / free mbarriers per slot
  __shared__ __align__(8) uint64_t bfull[RING];
  __shared__ __align__(8) uint64_t bfree[RING];
  __shared__ long long box_u[RING];
  __shared__ Acc box_v[RING];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  T* out = static_cast<T*>(a.out);
  Acc* partials = static_cast<Acc*>(a.partials);
  const int64_t S = a.Sr * a.Sc;
  const bool whole = (a.O == 1);
  const bool epi = !whole && S > 1;

  if (tid == 0) {
#pragma unroll
    for (int k = 0; k < NS; ++k) {
      mbar_init(&full[k], 1);
      mbar_init(&empty[k], kConsWarps);
    }
#pragma unroll
    for (int k = 0; k < RING; ++k) {
      mbar_init(&bfull[k], 1);
      mbar_init(&bfree[k], 1);
    }
    fence_mbar_init();
  }
  __syncthreads();
  pdl_wait();  // no global access above this line
  pdl_trigger();

  if (warp == 0) {
    // ---------------- producer warp: claims units, publishes their ids and
    // streams their 16-B aligned bodies into the ring NS stages ahead; it never
    // waits for the consumers' epilogues, only for a stage to be released.
    if (lane == 0) {
      tl_event(a.tl, TL_START, 0);
      int64_t g = 0;
      int seq = 0;
      // claims run two units ahead when units are short (guided tail phases
      // of one or two stages): a claim's L2 round trip then overlaps two
      // units' streaming instead of stalling the ring
      const bool deep = a.gd.nph > 1;
      long long u = claim_first(a.sched);
      long long n1 = deep ? claim_next(a.sched) : 0;
      while (true) {
        tl_event(a.tl, TL_UNIT, u);
        long long nu = claim_next(a.sched);  // next claim, in flight
        if (deep) {
          const long long t = n1;
          n1 = nu;
          nu = t;
        }
        const int slot0 = (int)(g % NS);
        s_units[seq & (RING - 1)] = u < a.units ? u : -1;
        ++seq;
        if (u >= a.units) {  // end marker: complete the next full phase without data
          if (g >= NS) mbar_wait(&empty[slot0], (unsigned)(((g / NS) - 1) & 1));
          mbar_arrive(&full[slot0]);
          break;
        }
        const StreamGeom geo = stream_geom<T>(a, u);
        const char* src = static_cast<const char*>(geo.row) + geo.head * (int64_t)sizeof(T);
        const int64_t bytes = geo.nbody * (int64_t)sizeof(T);
        const int64_t nk = (bytes + STAGE - 1) / STAGE;
        // RKR units are several rows at a stride: each stage is filled from
        // the concatenation of the unit's rows (one bulk copy per row piece)
        const int64_t rb = a.C > 1 ? a.L * (int64_t)sizeof(T) : bytes;
        const int64_t rs = a.rowStride * (int64_t)sizeof(T);
        int64_t r = 0, inrow = 0;
        for (int64_t k = 0; k < nk; ++k, ++g) {
          const int slot = (int)(g % NS);
          if (g >= NS) mbar_wait(&empty[slot], (unsigned)(((g / NS) - 1) & 1));
          const unsigned nb = (unsigned)min((int64_t)STAGE, bytes - k * STAGE);
          mbar_expect_tx(&full[slot], nb);
          for (unsigned done = 0; done < nb;) {
            const unsigned len = (unsigned)min((int64_t)(nb - done), rb - inrow);
            bulk_g2s(stage_mem + slot * STAGE + done, src + r * rs + inrow, len, &full[slot]);
            done += len;
            inrow += len;
            if (inrow == rb) { inrow = 0; ++r; }
          }
        }
        u = nu;
      }
      sched_exit(a.sched);
    }
    return;
  }
  if (warp == kConsWarps + 1) {
    // ---------------- epilogue warp (a4 per output): takes each unit's CTA
    // value from the mailbox, writes the unit partial, takes the output's
    // ticket, and the last arriver folds the output's S partials in unit
    // order.  The fence + atomic round trip no longer stalls the consumers
    // (r01y: 512^3 32-bit WV lost ~1 us of the whole CTA per unit).
    if (!epi) return;
    for (int n = 0;; ++n) {
      const int slot = n & (RING - 1);
      mbar_wait(&bfull[slot], (unsigned)((n / RING) & 1));
      const long long u = box_u[slot];
      const Acc v = box_v[slot];
      __syncwarp();
      if (lane == 0) mbar_arrive(&bfree[slot]);
      if (u < 0) break;
      int64_t o, sp;  // output and split of unit u (partials stay output-major)
      if (a.smaj && a.C > 1) {
        sp = u / a.O;
        o = u - sp * a.O;
      } else {
        o = u / S;
        sp = u - o * S;
      }
      unsigned t = 0;
      if (lane == 0) {
        partials[o * S + sp] = v;
        t = ticket_add(&a.tickets[o]);
      }
      t = __shfl_sync(0xffffffffu, t, 0);
      if (t == (unsigned)(S - 1)) {
        __threadfence();
        Acc w = fold_partials<OP, T>(partials + o * S, S, lane, 32);
        w = group_reduce<OP, T, 32>(w);
        if (lane == 0) {
          out[o] = merge_init<OP, T>(w, out, o, a.init_from_out);
          a.tickets[o] = 0u;
        }
      }
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
    for (int q = 0; q < VEC; ++q) acc[j][q] = O::identity();
  while (true) {
    // the first stage of the next unit (or the end marker) publishes its id
    mbar_wait(&full[g % NS], (unsigned)((g / NS) & 1));
    const long long u = s_units[seq & (RING - 1)];
    if (u < 0) break;
    const StreamGeom geo = stream_geom<T>(a, u);
    const T* row = static_cast<const T*>(geo.row);
    if (ct < geo.head) acc[0][0] = O::combine(acc[0][0], O::lift(ld_scalar(row + ct)));
    if (ct < geo.tail)
      acc[0][VEC - 1] = O::combine(acc[0][VEC - 1], O::lift(ld_scalar(row + geo.head + geo.nbody + ct)));
    const int64_t body_bytes = geo.nbody * (int64_t)sizeof(T);
    const int64_t nk = (body_bytes + STAGE - 1) / STAGE;
    for (int64_t k = 0; k < nk; ++k, ++g) {
      const int slot = (int)(g % NS);
      if (k > 0) mbar_wait(&full[slot], (unsigned)((g / NS) & 1));
      const int64_t bytes = min((int64_t)STAGE, body_bytes - k * STAGE);
      const unsigned char* st = stage_mem + slot * STAGE;
      if (bytes == STAGE) {  // full stage: all PER shared-memory loads in flight, then fold
        U128 x[PER];
#pragma unroll
        for (int j = 0; j < PER; ++j) x[j] = *reinterpret_cast<const U128*>(st + (ct + j * kConsThreads) * 16);
#pragma unroll
        for (int j = 0; j < PER; ++j)
#pragma unroll
          for (int q = 0; q < VEC; ++q) acc[j][q] = O::combine(acc[j][q], O::lift(unpack<T>(x[j], q)));
      } else {
#pragma unroll
        for (int j = 0; j < PER; ++j) {
          const int off = (ct + j * kConsThreads) * 16;
          if (off < bytes) {
            const U128 x = *reinterpret_cast<const U128*>(st + off);
#pragma unroll
            for (int q = 0; q < VEC; ++q) acc[j][q] = O::combine(acc[j][q], O::lift(unpack<T>(x, q)));
          }
        }
      }
      fence_proxy_async_smem();  // generic reads before the async refill
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[slot]);  // this warp is done with the stage
    }
    Acc v = fold_acc<OP, T, PER, VEC>(acc);
#pragma unroll
    for (int j = 0; j < PER; ++j)
#pragma unroll
      for (int q = 0; q < VEC; ++q) acc[j][q] = O::identity();
    // smem slots alternate between units: a warp can write unit n+2's slot
    // only after the barrier of unit n+1, i.e. after warp 0 read unit n's
    v = cons_reduce<OP, T>(v, smem + (seq & 1) * kConsWarps, cw, lane);
    const int64_t o = geo.o;
    if (ct == 0) tl_event(a.tl, TL_UNIT_DONE, u);
    if (whole) {
      if (ct == 0) partials[u] = v;
    } else if (S == 1) {
      if (ct == 0) out[o] = merge_init<OP, T>(v, out, o, a.init_from_out);
    } else if (ct == 0) {  // hand the unit to the epilogue warp
      const int slot = seq & (RING - 1);
      if (seq >= RING) mbar_wait(&bfree[slot], (unsigned)(((seq / RING) - 1) & 1));
      box_u[slot] = u;
      box_v[slot] = v;
      mbar_arrive(&bfull[slot]);
    }
    ++seq;
  }
  if (epi && ct == 0) {  // end marker for the epilogue warp
    const int slot = seq & (RING - 1);
    if (seq >= RING) mbar_wait(&bfree[slot], (unsigned)(((seq / RING) - 1) & 1));
    box_u[slot] = -1;
    mbar_arrive(&bfull[slot]);
  }
  if (ct == 0) tl_event(a.tl, TL_CONS_END, 0);
  if (whole) {  // a4: one ticket per CTA; the last CTA folds the S unit partials in unit order
    if (ct == 0) {
      const unsigned t = ticket_add(&a.tickets[0]);
      s_last = (t == gridDim.x - 1u);
    }
    cons_sync();
    if (s_last) {
      if (ct == 0) tl_event(a.tl, TL_FOLD, 0);
      __threadfence();
      Acc w = fold_partials_vec<OP, T>(partials, S, ct, kConsThreads);
      w = cons_reduce<OP, T>(w, smem, cw, lane);
      if (ct == 0) {
        const T r = merge_init<OP, T>(w, out, 0, a.init_from_out);
        a.tickets[0] = 0u;
        if (a.use_exch) peer_exchange<OP, T>(a.exch, out, r);
        else out[0] = r;
        tl_event(a.tl, TL_END, 0);
      }
    }
  }
}

// ------------------------------------------------------------- rows kernel
// KR with short rows (row_bytes a power of two in [512 B, 2 KiB], 16-B
// aligned): consecutive rows are one contiguous range, so a unit is a block of
// whole 16 KiB stages (RPS = 16 KiB / row_bytes >= 8 rows each), streamed by
// the producer warp with cp.async.bulk.  Consumer warp w owns rows
// w*RPW .. w*RPW+RPW-1 of every stage (RPW = RPS / 8): its lanes fold the
// row's 16-B vectors, one warp reduction (a2) per row, lane 0 writes the
// output (merging init).  No shared-memory combine and no barrier per stage
// (a first version with per-stage slot folds was consumer bound, r01), and
// rows never span CTAs, so there is no gang tier.
template <int OP, typename T, int NS>
__global__ void __launch_bounds__(kWsBlock) rows_kernel(SegArgs a) {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  constexpr int VEC = 16 / sizeof(T);
  constexpr int STAGE = kStageBytes;
  constexpr int RING = 8;
  extern __shared__ __align__(1024) unsigned char stage_mem[];  // NS * STAGE
  __shared__ __align__(8) uint64_t full[NS];
  __shared__ __align__(8) uint64_t empty[NS];
  __shared__ long long s_units[RING];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  T* out = static_cast<T*>(a.out);
  const int64_t row_bytes = a.L * (int64_t)sizeof(T);
  const int rshift = __ffsll(row_bytes) - 1;                 // row_bytes is a power of two
  const int rps = (int)(STAGE >> rshift);                     // rows per full stage
  const int64_t nst = (a.O + rps - 1) / rps;                  // stages overall
  const int64_t S = a.Sc;                                     // units (blocks of stages)

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
        const int64_t st0 = split_lo(nst, S, u), st1 = split_lo(nst, S, u + 1);
        for (int64_t st = st0; st < st1; ++st, ++g) {
          const int slot = (int)(g % NS);
          if (g >= NS) mbar_wait(&empty[slot], (unsigned)(((g / NS) - 1) & 1));
          const int64_t row0 = st * rps;
          const unsigned nb = (unsigned)(min((int64_t)rps, a.O - row0) << rshift);
          mbar_expect_tx(&full[slot], nb);
          bulk_g2s(stage_mem + slot * STAGE, static_cast<const char*>(a.in) + (row0 << rshift), nb, &full[slot]);
        }
        u = nu;
      }
      sched_exit(a.sched);
    }
    return;
  }

  // ---------------- consumer warps
  const int cw = warp - 1;
  int seq = 0;
  int64_t g = 0;
  while (true) {
    mbar_wait(&full[g % NS], (unsigned)((g / NS) & 1));
    const long long u = s_units[seq & (RING - 1)];
    if (u < 0) break;
    const int64_t st0 = split_lo(nst, S, u), st1 = split_lo(nst, S, u + 1);
    for (int64_t st = st0; st < st1; ++st, ++g) {
      const int slot = (int)(g % NS);
      if (st > st0) mbar_wait(&full[slot], (unsigned)((g / NS) & 1));
      const int64_t row0 = st * rps;
      const int nrows = (int)min((int64_t)rps, a.O - row0);
      const unsigned char* sm = stage_mem + slot * STAGE;
      const int rpw = rps / kConsWarps;                 // rows per warp (1, 2 or 4)
      const int vpl = (int)(row_bytes >> 9);            // 16-B vectors per lane per row (1..4)
      Acc v[4];
#pragma unroll
      for (int rr = 0; rr < 4; ++rr) {
        v[rr] = O::identity();
        const int r = cw * rpw + rr;
        if (rr < rpw && r < nrows) {
#pragma unroll
          for (int k = 0; k < 4; ++k) {
            if (k < vpl) {
              const U128 x = *reinterpret_cast<const U128*>(sm + ((int64_t)r << rshift) + (k * 32 + lane) * 16);
#pragma unroll
              for (int q = 0; q < VEC; ++q) v[rr] = O::combine(v[rr], O::lift(unpack<T>(x, q)));
            }
          }
        }
      }
      fence_proxy_async_smem();  // generic reads before the async refill
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[slot]);  // the stage is consumed into registers
#pragma unroll
      for (int rr = 0; rr < 4; ++rr) {
        if (rr < rpw) {  // warp-uniform
          const Acc w = group_reduce<OP, T, 32>(v[rr]);
          const int r = cw * rpw + rr;
          if (lane == 0 && r < nrows) {
            const int64_t o = row0 + r;
            out[o] = merge_init<OP, T>(w, out, o, a.init_from_out);
          }
        }
      }
    }
    ++seq;
  }
}

// ------------------------------------------------------------- flat column kernel
// RK / KRK with NARROW rows (row_bytes = K*size a power of two in [16, 4096] B,
// 16-B aligned): a CTA's load round (256 threads x 16 B = 4 KiB) covers whole
// rows, so thread t always meets the same column group (t*16 mod row_bytes)
// and a unit -- a block of whole rows of one batch -- is ONE contiguous range,
// streamed with fully coalesced 16-B loads (4 in flight per thread).  The
// worker tier folds the threads of each column group in shared memory (fixed
// order); the gang tier is the two-level ticket of coltma (unit partial rows
// of K values -> groups of kGroupFold -> batch).  The register column kernel
// left 1/2 to 31/32 of its lanes idle on such rows (r01: 1 TB/s on the
// paper's 2^20 x 2 x 32 gang case).
template <int OP, typename T>
__global__ void __launch_bounds__(kBlock, XR_SEG_MINB) colflat_kernel(const __grid_constant__ ColArgs a) {
  pdl_wait();  // no global access above this line
  pdl_trigger();
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  constexpr int VEC = 16 / sizeof(T);
  constexpr int U = kUnroll;
  __shared__ Acc red[kBlock][VEC];
  __shared__ int s_last;
  const int t = threadIdx.x;
  const int64_t row_bytes = a.K * (int64_t)sizeof(T);
  // 8-B rows (r02: two 32-bit columns): a 16-B vector holds two whole rows,
  // element q of every vector is column q % 2 -- one column group of VEC
  // lanes whose lanes fold into the K columns at the end
  const bool sub16 = sizeof(T) == 4 && row_bytes < 16;  // (compiled out for 8-byte types)
  const int G = sub16 ? 1 : (int)(row_bytes >> 4);  // 16-B column groups per row (1..256)
  const int64_t rp4k = 4096 / row_bytes;           // whole rows per (<= 4 KiB) load round
  // vectors per round (r02: rows of any multiple of 16 B, not only powers of
  // two): a round is rp4k whole rows, so thread t < NV always meets column
  // group t % G; threads >= NV idle (<= 6 % of the CTA)
  const int NV = sub16 ? kBlock : (int)(rp4k * G);  // (8-B rows: 512 rows = 256 vectors)
  const int64_t nblk = (a.R + rp4k - 1) / rp4k;    // 4 KiB row blocks per batch
  T* out = static_cast<T*>(a.out);
  Acc* partials = static_cast<Acc*>(a.partials);
  for (int64_t u = blockIdx.x; u < a.units; u += gridDim.x) {
    const int64_t b = u / a.S, s = u - b * a.S;
    const int64_t r0 = min(split_lo(nblk, a.S, s) * rp4k, a.R), r1 = min(split_lo(nblk, a.S, s + 1) * rp4k, a.R);
    const U128* __restrict__ base = reinterpret_cast<const U128*>(static_cast<const T*>(a.in) + (b * a.R + r0) * a.K);
    const int64_t nv = sub16 ? ((r1 - r0) >> 1) : (r1 - r0) * (row_bytes >> 4);  // whole 16-B vectors of the unit
    Acc acc[U][VEC];
#pragma unroll
    for (int k = 0; k < U; ++k)
#pragma unroll
      for (int q = 0; q < VEC; ++q) acc[k][q] = O::identity();
    int64_t v = t < NV ? t : nv;
    for (; v + (int64_t)(U - 1) * NV < nv; v += (int64_t)U * NV) {
      U128 x[U];
#pragma unroll
      for (int k = 0; k < U; ++k) x[k] = ld_stream(base + v + (int64_t)k * NV);
#pragma unroll
      for (int k = 0; k < U; ++k)
#pragma unroll
        for (int q = 0; q < VEC; ++q) acc[k][q] = O::combine(acc[k][q], O::lift(unpack<T>(x[k], q)));
    }
    for (; v < nv; v += NV) {
      const U128 x = ld_stream(base + v);
#pragma unroll
      for (int q = 0; q < VEC; ++q) acc[0][q] = O::combine(acc[0][q], O::lift(unpack<T>(x, q)));
    }
    if (sub16 && t == 0 && ((r1 - r0) * row_bytes) % 16 != 0) {  // an odd last 8-B row: lanes 0 .. K-1
      const T* last = static_cast<const T*>(a.in) + (b * a.R + r1 - 1) * a.K;
      for (int c = 0; c < (int)a.K; ++c) acc[0][c] = O::combine(acc[0][c], O::lift(ld_scalar(last + c)));
    }
#pragma unroll
    for (int k = 1; k < U; ++k)
#pragma unroll
      for (int q = 0; q < VEC; ++q) acc[0][q] = O::combine(acc[0][q], acc[k][q]);
#pragma unroll
    for (int q = 0; q < VEC; ++q) red[t][q] = acc[0][q];
    __syncthreads();
    // a3: column group g (< G) folds threads g, g+G, g+2G, ... in order; the
    // K = G*VEC unit results go to smem row red[0..G)
    Acc w[VEC];
    if (t < G) {
#pragma unroll
      for (int q = 0; q < VEC; ++q) w[q] = red[t][q];
      for (int m = t + G; m < NV; m += G)
#pragma unroll
        for (int q = 0; q < VEC; ++q) w[q] = O::combine(w[q], red[m][q]);
    }
    __syncthreads();
    if (t < G && !sub16) {
#pragma unroll
      for (int q = 0; q < VEC; ++q) reinterpret_cast<Acc*>(red)[t * VEC + q] = w[q];
    } else if (t == 0 && sub16) {  // lane q holds column q % K: fold the lanes per column, in lane order
      for (int c = 0; c < (int)a.K; ++c) {
        Acc z = w[c];
        for (int q = c + (int)a.K; q < VEC; q += (int)a.K) z = O::combine(z, w[q]);
        reinterpret_cast<Acc*>(red)[c] = z;
      }
    }
    __syncthreads();
    const Acc* col = reinterpret_cast<const Acc*>(red);  // col[c], c < K
    if (a.S == 1) {
      for (int c = t; c < a.K; c += kBlock) out[b * a.K + c] = merge_init<OP, T>(col[c], out, b * a.K + c, a.init_from_out);
    } else if (PackedAdd<OP, T>::value && a.packed) {  // a4 in one atomic per column (32-bit int '+')
      unsigned long long* pk = reinterpret_cast<unsigned long long*>(a.tickets) + b * a.K;
      for (int c = t; c < a.K; c += kBlock) {
        uint32_t sum;
        if (packed_add_arrive(pk + c, (uint32_t)col[c], a.S, &sum))
          out[b * a.K + c] = merge_init<OP, T>((Acc)sum, out, b * a.K + c, a.init_from_out);
      }
    } else {
      // a4, two levels over the S unit partial rows of batch b (K values each)
      Acc* P1 = partials + b * a.S * a.K;                         // [S][K]
      Acc* P2 = partials + a.B * a.S * a.K + b * a.G2 * a.K;      // [G2][K]
      unsigned* gt = a.tickets + b * a.G2;
      unsigned* tt = a.tickets + a.B * a.G2 + b;
      const int64_t gi = s / kGroupFold, g0 = gi * kGroupFold, gsz = min((int64_t)kGroupFold, a.S - g0);
      // fold rows [0, n) of a [n][K] partial block into column c; when K < the
      // CTA, kBlock / K row phases fold in parallel and meet in shared memory
      Acc* redf = reinterpret_cast<Acc*>(red);  // >= kBlock slots
      auto fold_rows = [&](const Acc* src, int64_t n, auto&& emit) {
        if (a.K < kBlock) {
          const int K = (int)a.K, nph = kBlock / K, c = t % K, ph = t / K;
          Acc z = O::identity();
          int64_t r = ph;
          for (; r + 3 * nph < n; r += 4 * nph) {
            Acc y[4];
#pragma unroll
            for (int k = 0; k < 4; ++k) y[k] = ld_partial(src + (r + k * nph) * a.K + c);
#pragma unroll
            for (int k = 0; k < 4; ++k) z = O::combine(z, y[k]);
          }
          for (; r < n; r += nph) z = O::combine(z, ld_partial(src + r * a.K + c));
          __syncthreads();  // redf may still be read (col) by other threads
          redf[ph * K + c] = z;
          __syncthreads();
          if (t < K) {
            Acc w2 = O::identity();
            for (int p2 = 0; p2 < nph; ++p2) w2 = O::combine(w2, redf[p2 * K + t]);
            emit(t, w2);
          }
        } else {
          for (int c = t; c < a.K; c += kBlock) {
            Acc z = O::identity();
            int64_t r = 0;
            for (; r + 3 < n; r += 4) {
              Acc y[4];
#pragma unroll
              for (int k = 0; k < 4; ++k) y[k] = ld_partial(src + (r + k) * a.K + c);
#pragma unroll
              for (int k = 0; k < 4; ++k) z = O::combine(z, y[k]);
            }
            for (; r < n; ++r) z = O::combine(z, ld_partial(src + r * a.K + c));
            emit(c, z);
          }
        }
      };
      for (int c = t; c < a.K; c += kBlock) P1[s * a.K + c] = col[c];
      __syncthreads();
      if (t == 0) {
        s_last = (ticket_add(&gt[gi]) == (unsigned)(gsz - 1));
      }
      __syncthreads();
      if (s_last) {
        __threadfence();
        auto to_out = [&](int c, Acc z) { out[b * a.K + c] = merge_init<OP, T>(z, out, b * a.K + c, a.init_from_out); };
        if (a.G2 == 1) {
          fold_rows(P1 + g0 * a.K, gsz, to_out);
          if (t == 0) gt[gi] = 0u;
        } else {
          fold_rows(P1 + g0 * a.K, gsz, [&](int c, Acc z) { P2[gi * a.K + c] = z; });
          __syncthreads();
          if (t == 0) {
            gt[gi] = 0u;
            s_last = (ticket_add(tt) == (unsigned)(a.G2 - 1));
          }
          __syncthreads();
          if (s_last) {
            __threadfence();
            fold_rows(P2, a.G2, to_out);
            if (t == 0) *tt = 0u;
          }
        }
      }
    }
    __syncthreads();
  }
}

// ------------------------------------------------------------- RKR rows kernel
// RKR (reduce outer k and inner i, keep the middle j) with short rows
// (row_bytes = L*size a power of two in [512 B, 2 KiB], 16-B aligned).  For a
// fixed k the rows (k, j) are contiguous, so J = 16 KiB / row_bytes
// consecutive outputs j form one 16 KiB stage.  A unit is (j-block jb, range
// of k): the producer warp streams the unit's stages (one cp.async.bulk per
// k, K*row_bytes apart in memory), and consumer warp w always
// meets the same rows -- outputs jb*J + w*rpw .. + rpw-1 -- in every stage,
// so its lanes accumulate them in registers across the whole k range with no
// shared-memory combine and no barrier per stage (the rows kernel's layout
// with a k loop).  At the end of a unit each warp reduces its rows (a2) and
// runs the per-output gang tier (a4): partials[j][s], a ticket per output,
// the last unit of output j folds its S partials.  (A first version streamed
// all rows and folded them by j into K-wide shared-memory partial rows: 0.60
// of peak, latency bound on the partial-row folds, r01.)
// Unit u -> (j-block, k split).  k-split-major (XR_RKR_KMAJOR=1): units that
// run at the same time read different j-blocks, i.e. different 16 KiB offsets
// within the 1 MiB k stride, instead of the same offset of many k planes.
#ifndef XR_RKR_KMAJOR
#define XR_RKR_KMAJOR 1
#endif
__device__ __forceinline__ void rkr_unit(int64_t u, int64_t S, int64_t njb, int64_t* jb, int64_t* s) {
#if XR_RKR_KMAJOR
  *s = u / njb;
  *jb = u - *s * njb;
#else
  *jb = u / S;
  *s = u - *jb * S;
#endif
}

// NARROW rows (16-256 B, r02): a stage holds J = 64-1024 rows, so consumer
// thread ct meets vectors ct + 256 i (i < 4) of every stage -- rows
// ct / vpr + i * (256 / vpr), always the same 4 outputs, piece ct % vpr --
// and accumulates them in registers across the k range; at the unit end the
// vpr threads of a row combine by shuffles and the row's leader runs the
// per-output gang tier itself (partial, ticket; the warp folds the outputs
// whose last split it holds).  The seg kernel read such rows 16-256 B at a
// time at the k stride: 0.7-1.5 TB/s (r02az).
template <typename Acc, int OP, typename T>
__device__ __forceinline__ Acc narrow_row_reduce(Acc v, int vpr) {
  switch (vpr) {
    case 1: return v;
    case 2: return group_reduce<OP, T, 2>(v);
    case 4: return group_reduce<OP, T, 4>(v);
    case 8: return group_reduce<OP, T, 8>(v);
    default: return group_reduce<OP, T, 16>(v);
  }
}

template <int OP, typename T, int NS, bool NARROW>
__global__ void __launch_bounds__(kWsEpiBlock, XR_WS_MINB) rkr_kernel(const __grid_constant__ RkrArgs a) {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  constexpr int VEC = 16 / sizeof(T);
  constexpr int STAGE = kStageBytes;
  constexpr int RING = 8;
  extern __shared__ __align__(1024) unsigned char stage_mem[];  // NS * STAGE
  __shared__ __align__(8) uint64_t full[NS];
  __shared__ __align__(8) uint64_t empty[NS];
  __shared__ long long s_units[RING];
  // per-output gang tier handed to the epilogue warp: a mailbox of RING units
  // (unit id + one value per output row of the j-block)
  __shared__ __align__(8) uint64_t bfull[RING];
  __shared__ __align__(8) uint64_t bfree[RING];
  __shared__ long long box_u[RING];
  __shared__ typename Op<OP, T>::Acc box_v[RING][32];
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  T* out = static_cast<T*>(a.out);
  const int64_t row_bytes = a.L * (int64_t)sizeof(T);
  const int rshift = __ffsll(row_bytes) - 1;  // row_bytes is a power of two (except NARROW rows)
  const int J = NARROW ? (int)(STAGE / row_bytes) : (int)(STAGE >> rshift);  // rows (outputs) per stage: 8, 16 or 32 (NARROW: 64..1024)
  const int64_t S = a.S;                       // k splits per j-block

  if (tid == 0) {
#pragma unroll
    for (int k = 0; k < NS; ++k) {
      mbar_init(&full[k], 1);
      mbar_init(&empty[k], kConsWarps);
    }
#pragma unroll
    for (int k = 0; k < RING; ++k) {
      mbar_init(&bfull[k], kConsWarps);
      mbar_init(&bfree[k], 1);
    }
    fence_mbar_init();
  }
  __syncthreads();
  pdl_wait();  // no global access above this line
  pdl_trigger();

  if (warp == 0) {  // ---------------- producer warp
    if (lane == 0) {
      int64_t g = 0;
      int seq = 0;
      long long u = claim_first(a.sched);
      while (true) {
        const long long nu = claim_next(a.sched);
        const int slot0 = (int)(g % NS);
        s_units[seq & (RING - 1)] = u < a.units ? u : -1;
        ++seq;
        if (u >= a.units) {
          if (g >= NS) mbar_wait(&empty[slot0], (unsigned)(((g / NS) - 1) & 1));
          mbar_arrive(&full[slot0]);
          break;
        }
        int64_t jb, s;
        rkr_unit(u, S, a.units / S, &jb, &s);
        const int64_t k0 = split_lo(a.C, S, s), k1 = split_lo(a.C, S, s + 1);
        // (NARROW rows need not be powers of two: multiply; the others shift)
        const unsigned nb = NARROW ? (unsigned)(min((int64_t)J, a.K - jb * J) * row_bytes)
                                   : (unsigned)(min((int64_t)J, a.K - jb * J) << rshift);
        const char* src = static_cast<const char*>(a.in) +
                          (NARROW ? (k0 * a.K + jb * J) * row_bytes : (k0 * a.K + jb * J) << rshift);
        const int64_t kstride = NARROW ? a.K * row_bytes : a.K << rshift;  // bytes between consecutive k
        for (int64_t k = k0; k < k1; ++k, ++g, src += kstride) {
          const int slot = (int)(g % NS);
          if (g >= NS) mbar_wait(&empty[slot], (unsigned)(((g / NS) - 1) & 1));
          mbar_expect_tx(&full[slot], nb);
          bulk_g2s(stage_mem + slot * STAGE, src, nb, &full[slot]);
        }
        u = nu;
      }
      sched_exit(a.sched);
    }
    return;
  }

  Acc* partials = static_cast<Acc*>(a.partials);
  if constexpr (NARROW) {
    if (warp == kConsWarps + 1) return;  // the consumers run the gang tier
    const int ct = tid - 32;
    const int vpr = (int)(row_bytes >> 4);  // 16-B vectors per row: 1..31
    // power-of-two rows: a row's vpr vectors sit in consecutive lanes of one
    // warp (shuffle combine); other multiples of 16 B: through shared memory
    const bool shfl = (vpr & (vpr - 1)) == 0;
    __shared__ Acc nsm[kConsThreads * 4];   // per-vector unit values (non-power-of-two rows)
    const int nvec = J * vpr;               // vectors of a full stage (<= 1024)
    int rowi[4];                            // row of my vector i of every stage
#pragma unroll
    for (int i = 0; i < 4; ++i) rowi[i] = (ct + i * kConsThreads) / vpr;
    const bool leader = shfl && (ct & (vpr - 1)) == 0;
    int seq = 0;
    int64_t g = 0;
    while (true) {
      mbar_wait(&full[g % NS], (unsigned)((g / NS) & 1));
      const long long u = s_units[seq & (RING - 1)];
      if (u < 0) break;
      int64_t jb, s;
      rkr_unit(u, S, a.units / S, &jb, &s);
      const int64_t k0 = split_lo(a.C, S, s), k1 = split_lo(a.C, S, s + 1);
      const int nrows = (int)min((int64_t)J, a.K - jb * J);
      Acc acc[4][VEC];
#pragma unroll
      for (int i = 0; i < 4; ++i)
#pragma unroll
        for (int q = 0; q < VEC; ++q) acc[i][q] = O::identity();
      for (int64_t k = k0; k < k1; ++k, ++g) {
        const int slot = (int)(g % NS);
        if (k > k0) mbar_wait(&full[slot], (unsigned)((g / NS) & 1));
        const unsigned char* sm = stage_mem + slot * STAGE;
        if (nrows == J && nvec == 4 * kConsThreads) {  // all 4 shared-memory loads in flight, then fold
          U128 x[4];
#pragma unroll
          for (int i = 0; i < 4; ++i) x[i] = *reinterpret_cast<const U128*>(sm + (ct + i * kConsThreads) * 16);
#pragma unroll
          for (int i = 0; i < 4; ++i)
#pragma unroll
            for (int q = 0; q < VEC; ++q) acc[i][q] = O::combine(acc[i][q], O::lift(unpack<T>(x[i], q)));
        } else {
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            if (ct + i * kConsThreads < nvec && rowi[i] < nrows) {
              const U128 x = *reinterpret_cast<const U128*>(sm + (ct + i * kConsThreads) * 16);
#pragma unroll
              for (int q = 0; q < VEC; ++q) acc[i][q] = O::combine(acc[i][q], O::lift(unpack<T>(x, q)));
            }
          }
        }
        fence_proxy_async_smem();  // generic reads before the async refill
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty[slot]);
      }
      // my 4 rows: combine, then (S > 1) store all 4 partials, ONE fence, and
      // the 4 tickets in flight together (one round trip, not four).  Power-
      // of-two rows: the row's vpr lanes combine by shuffles and the leader
      // lane owns the row; other rows: every vector's value goes to shared
      // memory and thread ct owns rows ct + 256 i, folding their vpr vectors
      // in order.
      Acc v[4];
      unsigned tk[4];
      int orow[4];      // the row thread ct owns in slot i, or -1
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        v[i] = acc[i][0];
#pragma unroll
        for (int q = 1; q < VEC; ++q) v[i] = O::combine(v[i], acc[i][q]);
      }
      if (shfl) {
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          v[i] = narrow_row_reduce<Acc, OP, T>(v[i], vpr);  // the row's vpr threads (lanes of one warp)
          orow[i] = (leader && rowi[i] < nrows) ? rowi[i] : -1;
        }
      } else {
#pragma unroll
        for (int i = 0; i < 4; ++i)
          if (ct + i * kConsThreads < nvec) nsm[ct + i * kConsThreads] = v[i];
        cons_sync();
#pragma unroll
        for (int i = 0; i < 4; ++i) {
          const int r = ct + i * kConsThreads;
          orow[i] = r < nrows ? r : -1;
          if (r < nrows) {
            Acc w = nsm[r * vpr];
            for (int p2 = 1; p2 < vpr; ++p2) w = O::combine(w, nsm[r * vpr + p2]);
            v[i] = w;
          }
        }
        cons_sync();  // nsm is rewritten at the next unit end
      }
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        if (orow[i] < 0) continue;
        const int64_t o = jb * J + orow[i];
        if (S == 1) out[o] = merge_init<OP, T>(v[i], out, o, a.init_from_out);
        else partials[o * S + s] = v[i];
      }
      if (S > 1) {
        __threadfence();
#pragma unroll
        for (int i = 0; i < 4; ++i)
          if (orow[i] >= 0) tk[i] = atomicAdd(&a.tickets[jb * J + orow[i]], 1u);
      }
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        if (S == 1) break;
        const int64_t o = jb * J + (orow[i] >= 0 ? orow[i] : 0);
        const bool last = orow[i] >= 0 && tk[i] == (unsigned)(S - 1);
        unsigned m = __ballot_sync(0xffffffffu, last);
        if (m) __threadfence();
        while (m) {  // the warp folds each output whose last split it holds, in split order
          const int l = __ffs(m) - 1;
          m &= m - 1;
          const int64_t ol = __shfl_sync(0xffffffffu, o, l);
          Acc w = fold_partials<OP, T>(partials + ol * S, S, lane, 32);
          w = group_reduce<OP, T, 32>(w);
          if (lane == 0) {
            out[ol] = merge_init<OP, T>(w, out, ol, a.init_from_out);
            a.tickets[ol] = 0u;
          }
        }
      }
      ++seq;
    }
    return;
  }
  if (warp == kConsWarps + 1) {
    // ---------------- epilogue warp (a4 per output, as in stream_kernel): lane
    // r takes row r's unit value, writes the partial and the output's ticket;
    // each output whose last unit this was is folded by the whole warp in
    // split order.  The consumers never wait for a fence + atomic round trip.
    if (S == 1) return;
    for (int n = 0;; ++n) {
      const int slot = n & (RING - 1);
      mbar_wait(&bfull[slot], (unsigned)((n / RING) & 1));
      const long long u = box_u[slot];
      if (u < 0) break;
      int64_t jb, s;
      rkr_unit(u, S, a.units / S, &jb, &s);
      const int nrows = (int)min((int64_t)J, a.K - jb * J);
      const Acc v = lane < nrows ? box_v[slot][lane] : O::identity();
      __syncwarp();
      if (lane == 0) mbar_arrive(&bfree[slot]);
      bool last = false;
      if (lane < nrows) {
        const int64_t o = jb * J + lane;
        partials[o * S + s] = v;
        last = (ticket_add(&a.tickets[o]) == (unsigned)(S - 1));
      }
      unsigned m = __ballot_sync(0xffffffffu, last);
      if (m) __threadfence();
      while (m) {
        const int r = __ffs(m) - 1;
        m &= m - 1;
        const int64_t o = jb * J + r;
        Acc w = fold_partials<OP, T>(partials + o * S, S, lane, 32);
        w = group_reduce<OP, T, 32>(w);
        if (lane == 0) {
          out[o] = merge_init<OP, T>(w, out, o, a.init_from_out);
          a.tickets[o] = 0u;
        }
      }
    }
    return;
  }

  // ---------------- consumer warps
  const int cw = warp - 1;
  const int rpw = J / kConsWarps;          // rows per warp per stage (1, 2 or 4)
  const int vpl = (int)(row_bytes >> 9);   // 16-B vectors per lane per row (1, 2 or 4)
  const int vsh = __ffs(vpl) - 1;          // rpw * vpl == 4: vector idx -> row idx >> vsh, piece idx & (vpl-1)
  int seq = 0;
  int64_t g = 0;
  while (true) {
    mbar_wait(&full[g % NS], (unsigned)((g / NS) & 1));
    const long long u = s_units[seq & (RING - 1)];
    if (u < 0) break;
    int64_t jb, s;
        rkr_unit(u, S, a.units / S, &jb, &s);
    const int64_t k0 = split_lo(a.C, S, s), k1 = split_lo(a.C, S, s + 1);
    const int nrows = (int)min((int64_t)J, a.K - jb * J);
    Acc acc[4][VEC];  // per vector idx (row idx >> vsh, piece idx & (vpl-1))
#pragma unroll
    for (int idx = 0; idx < 4; ++idx)
#pragma unroll
      for (int q = 0; q < VEC; ++q) acc[idx][q] = O::identity();
    const bool full_rows = (nrows == J);
    for (int64_t k = k0; k < k1; ++k, ++g) {
      const int slot = (int)(g % NS);
      if (k > k0) mbar_wait(&full[slot], (unsigned)((g / NS) & 1));
      const unsigned char* sm = stage_mem + slot * STAGE;
      if (full_rows) {  // all 4 shared-memory loads in flight, then fold
        U128 x[4];
#pragma unroll
        for (int idx = 0; idx < 4; ++idx)
          x[idx] = *reinterpret_cast<const U128*>(sm + ((int64_t)(cw * rpw + (idx >> vsh)) << rshift) +
                                                  ((idx & (vpl - 1)) * 32 + lane) * 16);
#pragma unroll
        for (int idx = 0; idx < 4; ++idx)
#pragma unroll
          for (int q = 0; q < VEC; ++q) acc[idx][q] = O::combine(acc[idx][q], O::lift(unpack<T>(x[idx], q)));
      } else {
#pragma unroll
        for (int idx = 0; idx < 4; ++idx) {
          const int r = cw * rpw + (idx >> vsh);
          if (r < nrows) {
            const U128 x = *reinterpret_cast<const U128*>(sm + ((int64_t)r << rshift) + ((idx & (vpl - 1)) * 32 + lane) * 16);
#pragma unroll
            for (int q = 0; q < VEC; ++q) acc[idx][q] = O::combine(acc[idx][q], O::lift(unpack<T>(x, q)));
          }
        }
      }
      fence_proxy_async_smem();  // generic reads before the async refill
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[slot]);  // the stage is consumed into registers
    }
    const int bslot = seq & (RING - 1);
    if (S > 1 && seq >= RING && lane == 0) mbar_wait(&bfree[bslot], (unsigned)(((seq / RING) - 1) & 1));
    __syncwarp();
#pragma unroll
    for (int rr = 0; rr < 4; ++rr) {
      const int r = cw * rpw + rr;
      if (rr < rpw && r < nrows) {  // warp-uniform
        Acc v = O::identity();
#pragma unroll
        for (int idx = 0; idx < 4; ++idx)
          if ((idx >> vsh) == rr)
#pragma unroll
            for (int q = 0; q < VEC; ++q) v = O::combine(v, acc[idx][q]);
        v = group_reduce<OP, T, 32>(v);
        const int64_t o = jb * J + r;
        if (S == 1) {
          if (lane == 0) out[o] = merge_init<OP, T>(v, out, o, a.init_from_out);
        } else if (lane == 0) {  // a4 runs in the epilogue warp
          box_v[bslot][r] = v;
        }
      }
    }
    if (S > 1 && lane == 0) {
      if (cw == 0) box_u[bslot] = u;
      mbar_arrive(&bfull[bslot]);
    }
    ++seq;
  }
  if (S > 1 && lane == 0) {  // end marker for the epilogue warp
    const int bslot = seq & (RING - 1);
    if (seq >= RING) mbar_wait(&bfree[bslot], (unsigned)(((seq / RING) - 1) & 1));
    if (cw == 0) box_u[bslot] = -1;
    mbar_arrive(&bfull[bslot]);
  }
}

// ------------------------------------------------------------- small whole-array kernel
// R shape on SMALL inputs (latency bound; e.g. the paper-style testsuite nest
// at gang+worker+vector, 2 MiB): ONE thread-block cluster of kClusterCtas
// CTAs x kClusterBlock threads; CTA r folds the contiguous r-th slice with 8
// 16-B loads in flight per thread (one load round at 2 MiB), a2 + a3 within
// the CTA, then the gang tier runs through DISTRIBUTED SHARED MEMORY: after a
// cluster barrier CTA 0 reads the CTAs' values in rank order and writes the
// output -- no global partials, no atomic ticket, no fence round trips (the
// seg kernel's last-CTA ticket chain costs ~2 us of a 4 us call).
template <int OP, typename T>
__global__ void __launch_bounds__(kClusterBlock) rcluster_kernel(const __grid_constant__ SegArgs a) {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  constexpr int VEC = 16 / sizeof(T);
  __shared__ Acc smem[32];
  __shared__ Acc cta_val;
  pdl_wait();  // no global access above this line
  pdl_trigger();
  const unsigned rank = blockIdx.x, nctas = gridDim.x;  // the grid is ONE cluster
  const int64_t c0 = split_lo_vec(a.L, nctas, rank, VEC), c1 = split_lo_vec(a.L, nctas, rank + 1, VEC);
  Acc acc[8][VEC];
#pragma unroll
  for (int k = 0; k < 8; ++k)
#pragma unroll
    for (int q = 0; q < VEC; ++q) acc[k][q] = O::identity();
  fold_row<OP, T, kClusterBlock, 8>(static_cast<const T*>(a.in) + c0, c1 - c0, threadIdx.x, acc);
  Acc v = fold_acc<OP, T, 8, VEC>(acc);
  v = block_reduce<OP, T, kClusterBlock>(v, smem);
  if (threadIdx.x == 0) cta_val = v;
  // cluster barrier (release / acquire): every CTA's value is visible in its
  // shared memory to the other CTAs of the cluster
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
  if (rank == 0 && threadIdx.x == 0) {
    Acc w = O::identity();
    const unsigned local = static_cast<unsigned>(__cvta_generic_to_shared(&cta_val));
#pragma unroll 1
    for (unsigned r = 0; r < nctas; ++r) {  // rank order: deterministic
      unsigned remote;
      asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(remote) : "r"(local), "r"(r));
      Acc x;
      if constexpr (sizeof(Acc) == 4) {
        unsigned b;
        asm volatile("ld.shared::cluster.u32 %0, [%1];" : "=r"(b) : "r"(remote) : "memory");
        memcpy(&x, &b, 4);
      } else {
        unsigned long long b;
        asm volatile("ld.shared::cluster.u64 %0, [%1];" : "=l"(b) : "r"(remote) : "memory");
        memcpy(&x, &b, 8);
      }
      w = O::combine(w, x);
    }
    T* out = static_cast<T*>(a.out);
    out[0] = merge_init<OP, T>(w, out, 0, a.init_from_out);
  }
  // keep every CTA's shared memory alive until CTA 0 has read it
  asm volatile("barrier.cluster.arrive.release.aligned;\n\tbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}

// ------------------------------------------------------------- small column kernel
// RK / KRK on SMALL inputs (latency bound, e.g. the paper-style testsuite nest
// 64 x 64 x 128 at gang or worker level) with few reduced rows (R <= 256):
// one WARP per group of CW = 32 B of kept columns; lane l folds rows l, l+32,
// ... (two 16-B loads per row, four in flight), then one warp reduction per
// column (a2: REDUX / shuffles) and lanes 0..CW-1 write the CW outputs.  No
// shared memory, no barrier and no gang tier, and 8x more CTAs than the
// CTA-per-tile column kernels (r01: 64 CTAs of 32 KiB for cfg1 G / W, 5.3 us
// graph-replayed, vs 2.1 us for the 512-CTA row case).
template <int OP, typename T>
__global__ void __launch_bounds__(kBlock) colsmall_kernel(const __grid_constant__ ColArgs a) {
  pdl_wait();  // no global access above this line
  pdl_trigger();
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  constexpr int VEC = 16 / sizeof(T);
  constexpr int CW = 2 * VEC;  // columns per warp
  const int lane = threadIdx.x & 31;
  const int64_t gw = ((int64_t)blockIdx.x * kBlock + threadIdx.x) >> 5;
  if (gw >= a.units) return;  // warp-uniform
  const int64_t b = gw / a.tiles, c0 = (gw - b * a.tiles) * CW;
  const bool two = c0 + CW <= a.K;  // else only the first vector (K % VEC == 0)
  const T* __restrict__ base = static_cast<const T*>(a.in) + b * a.R * a.K + c0;
  T* out = static_cast<T*>(a.out);
  Acc acc[CW];
#pragma unroll
  for (int q = 0; q < CW; ++q) acc[q] = O::identity();
  int64_t r = lane;
  for (; r + 32 < a.R; r += 64) {  // two rows, four 16-B loads in flight
    const T* p0 = base + r * a.K;
    const T* p1 = p0 + 32 * a.K;
    const U128 x0 = ld_stream(p0), x2 = ld_stream(p1);
    U128 x1 = x0, x3 = x2;
    if (two) { x1 = ld_stream(p0 + VEC); x3 = ld_stream(p1 + VEC); }
#pragma unroll
    for (int q = 0; q < VEC; ++q) {
      acc[q] = O::combine(acc[q], O::lift(unpack<T>(x0, q)));
      acc[q] = O::combine(acc[q], O::lift(unpack<T>(x2, q)));
      if (two) {
        acc[VEC + q] = O::combine(acc[VEC + q], O::lift(unpack<T>(x1, q)));
        acc[VEC + q] = O::combine(acc[VEC + q], O::lift(unpack<T>(x3, q)));
      }
    }
  }
  if (r < a.R) {
    const T* p0 = base + r * a.K;
    const U128 x0 = ld_stream(p0);
    U128 x1 = x0;
    if (two) x1 = ld_stream(p0 + VEC);
#pragma unroll
    for (int q = 0; q < VEC; ++q) {
      acc[q] = O::combine(acc[q], O::lift(unpack<T>(x0, q)));
      if (two) acc[VEC + q] = O::combine(acc[VEC + q], O::lift(unpack<T>(x1, q)));
    }
  }
  Acc mine = O::identity();
#pragma unroll
  for (int q = 0; q < CW; ++q) {
    const Acc v = group_reduce<OP, T, 32>(acc[q]);
    if (lane == q) mine = v;
  }
  if (lane < (two ? CW : VEC)) {
    const int64_t o = b * a.K + c0 + lane;
    out[o] = merge_init<OP, T>(mine, out, o, a.init_from_out);
  }
}

// ------------------------------------------------------------- col kernel
// Lanes own VEC contiguous kept columns (a 32*VEC-column tile per warp row);
// the CTA's warps stride over the reduced rows of a row chunk; the worker tier
// is a cross-warp combine of per-column partials in shared memory.
template <int OP, typename T, int VEC, int BLOCK, int U>
// (the column kernel keeps its 16-B loads batched with min 1, not 4 -- SASS guard)
#ifndef XR_COL_MINB
#define XR_COL_MINB 1
#endif
__global__ void __launch_bounds__(BLOCK, XR_COL_MINB) col_kernel(const __grid_constant__ ColArgs a) {
  pdl_wait();  // no global access above this line
  pdl_trigger();
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  constexpr int NW = BLOCK / 32;
  constexpr int TW = 32 * VEC;
  static_assert(TW <= BLOCK, "tile wider than the CTA");
  __shared__ Acc sm[NW][TW];
  __shared__ int s_last;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, t = threadIdx.x;
  const T* __restrict__ in = static_cast<const T*>(a.in);
  T* out = static_cast<T*>(a.out);
  Acc* partials = static_cast<Acc*>(a.partials);
  const int64_t per_b = a.tiles * a.S;

  __shared__ long long s_unit[2];
  if (t == 0) s_unit[0] = claim_first(a.sched);
  __syncthreads();
  long long u = s_unit[0];
  int par = 1;
  while (u < a.units) {
    if (t == 0) s_unit[par] = claim_next(a.sched);  // next unit, in flight
    const int64_t b = u / per_b, rem = u - b * per_b;
    const int64_t tile = rem / a.S, s = rem - tile * a.S;
    const int64_t col = tile * TW + (int64_t)lane * VEC;
    const int64_t r0 = split_lo(a.R, a.S, s), r1 = split_lo(a.R, a.S, s + 1);
    Acc acc[U][VEC];
#pragma unroll
    for (int k = 0; k < U; ++k)
#pragma unroll
      for (int q = 0; q < VEC; ++q) acc[k][q] = O::identity();
    if (col < a.K) {  // VEC path: K % VEC == 0, so the lane owns VEC whole columns
      const T* __restrict__ base = in + b * a.R * a.K + col;
      int64_t r = r0 + warp;
      if constexpr (VEC > 1) {
        for (; r + (int64_t)(U - 1) * NW < r1; r += (int64_t)U * NW) {
          U128 x[U];
#pragma unroll
          for (int k = 0; k < U; ++k) x[k] = ld_stream(base + (r + (int64_t)k * NW) * a.K);
#pragma unroll
          for (int k = 0; k < U; ++k)
#pragma unroll
            for (int q = 0; q < VEC; ++q) acc[k][q] = O::combine(acc[k][q], O::lift(unpack<T>(x[k], q)));
        }
        for (; r < r1; r += NW) {
          const U128 x = ld_stream(base + r * a.K);
#pragma unroll
          for (int q = 0; q < VEC; ++q) acc[0][q] = O::combine(acc[0][q], O::lift(unpack<T>(x, q)));
        }
      } else {
        for (; r + (int64_t)(U - 1) * NW < r1; r += (int64_t)U * NW) {
          T x[U];
#pragma unroll
          for (int k = 0; k < U; ++k) x[k] = ld_scalar(base + (r + (int64_t)k * NW) * a.K);
#pragma unroll
          for (int k = 0; k < U; ++k) acc[k][0] = O::combine(acc[k][0], O::lift(x[k]));
        }
        for (; r < r1; r += NW) acc[0][0] = O::combine(acc[0][0], O::lift(ld_scalar(base + r * a.K)));
      }
    }
#pragma unroll
    for (int k = 1; k < U; ++k)
#pragma unroll
      for (int q = 0; q < VEC; ++q) acc[0][q] = O::combine(acc[0][q], acc[k][q]);
#pragma unroll
    for (int q = 0; q < VEC; ++q) sm[warp][lane * VEC + q] = acc[0][q];
    __syncthreads();
    // a3: worker tier, fixed warp order per column
    Acc v = O::identity();
    if (t < TW) {
#pragma unroll
      for (int w = 0; w < NW; ++w) v = O::combine(v, sm[w][t]);
    }
    const int64_t oc = tile * TW + t;
    if (a.S == 1) {
      if (t < TW && oc < a.K) out[b * a.K + oc] = merge_init<OP, T>(v, out, b * a.K + oc, a.init_from_out);
    } else {  // a4: gang tier per column tile
      Acc* P = partials + (b * a.tiles + tile) * a.S * TW;
      if (t < TW) P[s * TW + t] = v;
      __syncthreads();  // the CTA's partial stores happen-before thread 0's fence (cumulative)
      if (t == 0) {
        const unsigned tk = ticket_add(&a.tickets[b * a.tiles + tile]);
        s_last = (tk == (unsigned)(a.S - 1));
      }
      __syncthreads();
      if (s_last) {
        __threadfence();
        Acc w2[VEC];
#pragma unroll
        for (int q = 0; q < VEC; ++q) w2[q] = O::identity();
        int64_t si = warp;
        for (; si + 3 * NW < a.S; si += 4 * NW) {
          Acc y[4][VEC];
#pragma unroll
          for (int k = 0; k < 4; ++k)
#pragma unroll
            for (int q = 0; q < VEC; ++q) y[k][q] = ld_partial(P + (si + k * NW) * TW + lane * VEC + q);
#pragma unroll
          for (int k = 0; k < 4; ++k)
#pragma unroll
            for (int q = 0; q < VEC; ++q) w2[q] = O::combine(w2[q], y[k][q]);
        }
        for (; si < a.S; si += NW)
#pragma unroll
          for (int q = 0; q < VEC; ++q) w2[q] = O::combine(w2[q], ld_partial(P + si * TW + lane * VEC + q));
#pragma unroll
        for (int q = 0; q < VEC; ++q) sm[warp][lane * VEC + q] = w2[q];
        __syncthreads();
        if (t < TW) {
          Acc z = O::identity();
#pragma unroll
          for (int w = 0; w < NW; ++w) z = O::combine(z, sm[w][t]);
          if (oc < a.K) out[b * a.K + oc] = merge_init<OP, T>(z, out, b * a.K + oc, a.init_from_out);
        }
        if (t == 0) a.tickets[b * a.tiles + tile] = 0u;
      }
    }
    __syncthreads();
    u = s_unit[par];
    par ^= 1;
  }
  sched_exit(a.sched);
}

// ------------------------------------------------------------- col TMA kernel
// RK / KRK with 16-B aligned rows of >= 1 KiB: a 3-D TMA tensor map over
// (K, R, B) loads boxes of 1 KiB x kColBoxRows rows into the shared-memory
// ring (cp.async.bulk.tensor, SASS UTMALDG), thread 0 producing NS boxes ahead
// across unit boundaries.  Threads own a 16-B column group and a row phase;
// the worker tier folds the row phases per column in shared memory; the gang
// tier is the per-tile ticket of col_kernel.  OOB rows/columns of a box are
// skipped by the consumers, so the fill value never matters.
// Deferred group tickets: consumer thread 0 resolves a unit's group ticket at
// the end of the NEXT unit, so the consumers do not wait for the fence +
// atomic round trip.  MEASURED SLOWER (r02 same-box A/B: 512^3 32-bit G 86.5
// vs 84.5 us, GW 93.3 vs 90.6 us; the delayed group folds lengthen the end of
// the launch), so the ticket is resolved at once by default.
#ifndef XR_COLTMA_DEFER
#define XR_COLTMA_DEFER 0
#endif
template <int OP, typename T, int NS, int BW>  // BW: box width in bytes (one box row)
__global__ void __launch_bounds__(kWsBlock, XR_WS_MINB) coltma_kernel(const __grid_constant__ CUtensorMap tmap, ColArgs a) {
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  constexpr int BLOCK = kConsThreads;        // consumer threads
  constexpr int VEC = 16 / sizeof(T);
  constexpr int TW = BW / (int)sizeof(T);    // box columns
  constexpr int BR = kStageBytes / BW;       // box rows
  constexpr int G = TW / VEC;                // 16-B column groups per row
  constexpr int NPH = BLOCK / G;             // row phases
  constexpr int RING = 8;
  constexpr int AV = 16 / (int)sizeof(Acc);  // partials per 16-B load in the folds
  constexpr int NPA = BLOCK / (TW / AV);     // row phases of the folds
  constexpr int NRED = NPH > NPA ? NPH : NPA;
  static_assert(NPH >= 1 && NPA >= 1 && BR % NPH == 0, "geometry");
  extern __shared__ __align__(1024) unsigned char stage_mem[];  // NS * kStageBytes
  __shared__ __align__(8) uint64_t full[NS];
  __shared__ __align__(8) uint64_t empty[NS];
  __shared__ long long s_units[RING];
  __shared__ __align__(16) Acc red[NRED][TW];
  __shared__ int s_last;
  const int tid0 = threadIdx.x, warp = tid0 >> 5, lane = tid0 & 31;
  T* out = static_cast<T*>(a.out);
  Acc* partials = static_cast<Acc*>(a.partials);
  const int64_t per_b = a.tiles * a.S;
  // unit id -> (batch, tile, split): tile-major (the splits of one tile are
  // consecutive ids) or split-major (a.smaj: concurrently claimed units cover
  // every tile of the same row range -- one moving window of the array)
  auto decode = [&](long long u, int64_t* b, int64_t* tile, int64_t* s) {
    if (a.smaj) {
      const int64_t bt = a.B * a.tiles;
      *s = u / bt;
      const int64_t r = u - *s * bt;
      *b = r / a.tiles;
      *tile = r - *b * a.tiles;
    } else {
      *b = u / per_b;
      const int64_t rem = u - *b * per_b;
      *tile = rem / a.S;
      *s = rem - *tile * a.S;
    }
  };

  if (tid0 == 0) {
    asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&tmap)) : "memory");
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

  if (warp == 0) {
    // ---------------- producer warp
    if (lane == 0) {
      tl_event(a.tl, TL_START, 0);
      int64_t g = 0;
      int seq = 0;
      long long u = claim_first(a.sched);
      while (true) {
        tl_event(a.tl, TL_UNIT, u);
        const long long nu = claim_next(a.sched);
        const int slot0 = (int)(g % NS);
        s_units[seq & (RING - 1)] = u < a.units ? u : -1;
        ++seq;
        if (u >= a.units) {
          if (g >= NS) mbar_wait(&empty[slot0], (unsigned)(((g / NS) - 1) & 1));
          mbar_arrive(&full[slot0]);
          break;
        }
        int64_t b, tile, s;
        decode(u, &b, &tile, &s);
        int64_t r0, r1;
        box_rows(a.R, a.S, s, BR, &r0, &r1);
        const int64_t nk = (r1 - r0 + BR - 1) / BR;
        for (int64_t k = 0; k < nk; ++k, ++g) {
          const int slot = (int)(g % NS);
          if (g >= NS) mbar_wait(&empty[slot], (unsigned)(((g / NS) - 1) & 1));
          mbar_expect_tx(&full[slot], (unsigned)kStageBytes);
          tma_load_3d(stage_mem + slot * kStageBytes, &tmap, (int)(tile * TW), (int)(r0 + k * BR), (int)b,
                      &full[slot]);
        }
        u = nu;
      }
      sched_exit(a.sched);
    }
    return;
  }

  // ---------------- consumer warps
  const int tid = tid0 - 32, grp = tid % G, ph = tid / G;
  int seq = 0;
  int64_t g = 0;
  // fold rows [0, n) of a [n][TW] partial block into column tid (< TW):
  // 16-B L2 loads, NPA row phases x (TW/AV) column groups, 4 rows in flight
  auto fold_rows = [&](const Acc* base, int64_t n) -> Acc {
    const int cg = tid % (TW / AV), q2 = tid / (TW / AV);
    Acc w[AV];
#pragma unroll
    for (int q = 0; q < AV; ++q) w[q] = O::identity();
    int64_t r = q2;
    for (; r + 3 * NPA < n; r += 4 * NPA) {
      uint4 y[4];
#pragma unroll
      for (int k = 0; k < 4; ++k) y[k] = __ldcg(reinterpret_cast<const uint4*>(base + (r + k * NPA) * TW + cg * AV));
#pragma unroll
      for (int k = 0; k < 4; ++k)
#pragma unroll
        for (int q = 0; q < AV; ++q) w[q] = O::combine(w[q], reinterpret_cast<const Acc*>(&y[k])[q]);
    }
    for (; r < n; r += NPA) {
      const uint4 y = __ldcg(reinterpret_cast<const uint4*>(base + r * TW + cg * AV));
#pragma unroll
      for (int q = 0; q < AV; ++q) w[q] = O::combine(w[q], reinterpret_cast<const Acc*>(&y)[q]);
    }
#pragma unroll
    for (int q = 0; q < AV; ++q) red[q2][cg * AV + q] = w[q];
    cons_sync();
    Acc z = O::identity();
    if (tid < TW) {
#pragma unroll
      for (int p2 = 0; p2 < NPA; ++p2) z = O::combine(z, red[p2][tid]);
    }
    return z;
  };
  // a4, two levels: unit partial -> group of a.gf (its last unit folds
  // the group in unit order) -> tile (the last group folds the G2 group
  // partials).  The group ticket of a unit is DEFERRED: consumer thread 0
  // issues the fence + atomic after the unit's partial store and the
  // consumers go straight on to the next unit; the returned ticket is read
  // (and, if this unit was its group's last, the group folded) at the end of
  // the next unit or after the loop.  The consumers no longer wait for the
  // fence + atomic round trip of every unit (r01: each unit stalled all 8
  // consumer warps ~1 us; more, shorter units were then a net loss).
  unsigned pend_tk = 0u;   // consumer thread 0: ticket value of the pending unit
  long long pend_u = -1;   // the pending unit (uniform across consumers)
  auto finish_pending = [&]() {
    if (pend_u < 0) return;
    int64_t b, tile, s;
    decode(pend_u, &b, &tile, &s);
    const int64_t tid_tile = b * a.tiles + tile;
    const int64_t grp_i = s / a.gf;
    const int64_t g0 = grp_i * a.gf, gsz = min((int64_t)a.gf, a.S - g0);
    if (tid == 0) s_last = (pend_tk == (unsigned)(gsz - 1));
    cons_sync();
    pend_u = -1;
    if (!s_last) return;  // uniform
    Acc* P1 = partials + tid_tile * a.S * TW;                                  // [S][TW]
    Acc* P2 = partials + a.B * a.tiles * a.S * TW + tid_tile * a.G2 * TW;      // [G2][TW]
    unsigned* gt = a.tickets + tid_tile * a.G2;                                // group tickets
    unsigned* tt = a.tickets + a.B * a.tiles * a.G2 + tid_tile;                // tile ticket
    const int64_t oc = tile * TW + tid;
    __threadfence();
    const Acc w = fold_rows(P1 + g0 * TW, gsz);
    if (tid == 0) gt[grp_i] = 0u;
    if (a.G2 == 1) {
      if (tid < TW && oc < a.K) out[b * a.K + oc] = merge_init<OP, T>(w, out, b * a.K + oc, a.init_from_out);
    } else {
      if (tid < TW) P2[grp_i * TW + tid] = w;
      cons_sync();
      if (tid == 0) {
        const unsigned tk = ticket_add(tt);
        s_last = (tk == (unsigned)(a.G2 - 1));
      }
      cons_sync();
      if (s_last) {
        __threadfence();
        const Acc z = fold_rows(P2, a.G2);
        if (tid < TW && oc < a.K) out[b * a.K + oc] = merge_init<OP, T>(z, out, b * a.K + oc, a.init_from_out);
        if (tid == 0) *tt = 0u;
      }
    }
    cons_sync();  // red is reused
  };
  while (true) {
    mbar_wait(&full[g % NS], (unsigned)((g / NS) & 1));
    const long long u = s_units[seq & (RING - 1)];
    if (u < 0) break;
    int64_t b, tile, s;
    decode(u, &b, &tile, &s);
    int64_t r0, r1;
    box_rows(a.R, a.S, s, BR, &r0, &r1);
    const int64_t nk = (r1 - r0 + BR - 1) / BR;
    const bool col_ok = tile * TW + (int64_t)grp * VEC < a.K;  // K % VEC == 0: whole vectors
    Acc acc[2][VEC];
#pragma unroll
    for (int j = 0; j < 2; ++j)
#pragma unroll
      for (int q = 0; q < VEC; ++q) acc[j][q] = O::identity();
    for (int64_t k = 0; k < nk; ++k, ++g) {
      const int slot = (int)(g % NS);
      if (k > 0) mbar_wait(&full[slot], (unsigned)((g / NS) & 1));
      const unsigned char* st = stage_mem + slot * kStageBytes;
      const int64_t rbase = r0 + k * BR;
      if (col_ok && rbase + BR <= r1) {  // full box: all BR / NPH loads in flight, then fold
        U128 x[BR / NPH];
#pragma unroll
        for (int i = 0; i < BR / NPH; ++i) x[i] = *reinterpret_cast<const U128*>(st + (ph + i * NPH) * BW + grp * 16);
#pragma unroll
        for (int i = 0; i < BR / NPH; ++i)
#pragma unroll
          for (int q = 0; q < VEC; ++q) acc[i & 1][q] = O::combine(acc[i & 1][q], O::lift(unpack<T>(x[i], q)));
      } else {
#pragma unroll
        for (int i = 0; i < BR / NPH; ++i) {
          const int row = ph + i * NPH;
          if (col_ok && rbase + row < r1) {
            const U128 x = *reinterpret_cast<const U128*>(st + row * BW + grp * 16);
#pragma unroll
            for (int q = 0; q < VEC; ++q) acc[i & 1][q] = O::combine(acc[i & 1][q], O::lift(unpack<T>(x, q)));
          }
        }
      }
      fence_proxy_async_smem();  // generic reads before the async refill
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[slot]);
    }
    // a3: fold the row phases per column
#pragma unroll
    for (int q = 0; q < VEC; ++q) red[ph][grp * VEC + q] = O::combine(acc[0][q], acc[1][q]);
    cons_sync();
    const int64_t oc = tile * TW + tid;  // output column of thread tid (< TW)
    Acc v = O::identity();
    if (tid < TW) {
#pragma unroll
      for (int p2 = 0; p2 < NPH; ++p2) v = O::combine(v, red[p2][tid]);
    }
    if (tid == 0) tl_event(a.tl, TL_UNIT_DONE, u);
    if (a.S == 1) {
      if (tid < TW && oc < a.K) out[b * a.K + oc] = merge_init<OP, T>(v, out, b * a.K + oc, a.init_from_out);
      cons_sync();  // red is reused by the next unit
    } else {
      const int64_t tid_tile = b * a.tiles + tile;
      Acc* P1 = partials + tid_tile * a.S * TW;  // [S][TW]
      if (tid < TW) P1[s * TW + tid] = v;
      cons_sync();  // partial stores happen-before thread 0's (cumulative) fence; red free
      finish_pending();  // the previous unit's group (its ticket has long returned)
      if (tid == 0) pend_tk = ticket_add(&a.tickets[tid_tile * a.G2 + s / a.gf]);  // result read later
      pend_u = u;
#if !XR_COLTMA_DEFER
      finish_pending();  // A/B: resolve the ticket right away (the r01 behaviour)
#endif
    }
    ++seq;
  }
  if (tid == 0) tl_event(a.tl, TL_CONS_END, 0);
  finish_pending();
  if (tid == 0) tl_event(a.tl, TL_END, 0);
}

// ------------------------------------------------------------- short-row kernel
// KR with SHORT power-of-two rows (4-128 B, 16-B aligned input; r02): every
// thread takes one CH-byte chunk (CH = max(64 B, row)) of whole rows per
// round -- CH / 16 vector loads in flight -- folds each row in element order
// and writes its CH / row_bytes outputs; adjacent threads hold adjacent
// chunks, so loads and stores are coalesced.  The seg kernel's 8-lane groups
// reduced one such row per group and round: 8 B rows at 0.14 TB/s (r02bk).
template <int OP, typename T, int CH>
__global__ void __launch_bounds__(kBlock) shortrow_kernel(const __grid_constant__ SegArgs a) {
  pdl_wait();  // no global access above this line
  pdl_trigger();
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  constexpr int VEC = 16 / (int)sizeof(T);
  constexpr int NVC = CH / 16;                 // vectors per chunk
  constexpr int E = CH / (int)sizeof(T);       // elements per chunk
  // the block's outputs are staged in shared memory and stored as 16-B
  // vectors (r02bq: 8 scalar stores per thread, 32 B apart across a warp,
  // bound 8-B rows at 28 % of DRAM peak)
  __shared__ __align__(16) T so[kBlock * (E / 2)];
  const T* in = static_cast<const T*>(a.in);
  T* out = static_cast<T*>(a.out);
  const int L = (int)a.L;                      // elements per row (power of two, <= E)
  const int rpt = E / L;                       // rows per chunk
  const int64_t nchunks = a.O / rpt;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  const int64_t t0 = (int64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const bool vst = ((uintptr_t)out & 15u) == 0;
  // staging pays only when a thread holds several rows (r02br: one row per
  // thread -- a warp's outputs already contiguous -- was 7-16 % slower staged)
  const bool stage = rpt >= 2;
  for (int64_t cb = (int64_t)blockIdx.x * blockDim.x; cb < nchunks; cb += stride) {  // block-uniform
    const int64_t c = cb + threadIdx.x;
    if (c < nchunks) {
      const U128* p = reinterpret_cast<const U128*>(in + c * E);
      U128 x[NVC];
#pragma unroll
      for (int v = 0; v < NVC; ++v) x[v] = ld_stream(p + v);
      Acc acc = O::identity();
#pragma unroll
      for (int e = 0; e < E; ++e) {
        acc = O::combine(acc, O::lift(unpack<T>(x[e / VEC], e % VEC)));
        if (((e + 1) & (L - 1)) == 0) {  // row e / L complete
          const int64_t o = c * rpt + e / L;
          const T r = merge_init<OP, T>(acc, out, o, a.init_from_out);
          if (stage) so[threadIdx.x * rpt + e / L] = r;
          else out[o] = r;
          acc = O::identity();
        }
      }
    }
    if (!stage) continue;  // (block-uniform)
    __syncthreads();
    const int64_t nb = min((int64_t)blockDim.x, nchunks - cb) * rpt;  // outputs of this block round
    T* ob = out + cb * rpt;                                              // 16-B aligned when out is
    int64_t done = 0;
    if (vst) {
      for (int64_t i = threadIdx.x; i < nb / VEC; i += blockDim.x)
        *reinterpret_cast<U128*>(ob + i * VEC) = *reinterpret_cast<const U128*>(so + i * VEC);
      done = nb / VEC * VEC;
    }
    for (int64_t i = done + threadIdx.x; i < nb; i += blockDim.x) ob[i] = so[i];
    __syncthreads();  // so is rewritten by the next round
  }
  // rows of the last partial chunk: one thread per row, in element order
  for (int64_t o = nchunks * rpt + t0; o < a.O; o += stride) {
    Acc acc = O::identity();
    for (int i = 0; i < L; ++i) acc = O::combine(acc, O::lift(ld_scalar(in + o * L + i)));
    out[o] = merge_init<OP, T>(acc, out, o, a.init_from_out);
  }
}

// ------------------------------------------------------------- thin column kernel
// RK / KRK with FEW reduced rows (R <= 32) and many kept columns, 16-B
// aligned rows (r02): the output is as large as the input, so each thread
// owns one 16-B column group, folds its R rows in order (4 loads in flight)
// and stores VEC outputs -- an elementwise-style pass.  The column kernels'
// tiles and splits cost a full unit per 2-16 rows there (r02bk: R = 2 rows
// of 256 MiB in 874 us).
template <int OP, typename T>
__global__ void __launch_bounds__(kBlock) thincol_kernel(const __grid_constant__ ColArgs a) {
  pdl_wait();  // no global access above this line
  pdl_trigger();
  using O = Op<OP, T>;
  using Acc = typename O::Acc;
  constexpr int VEC = 16 / (int)sizeof(T);
  const T* in = static_cast<const T*>(a.in);
  T* out = static_cast<T*>(a.out);
  const int64_t gpr = a.K / VEC;  // 16-B column groups per row
  const int64_t ng = a.B * gpr;
  const int R = (int)a.R;
  for (int64_t c = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; c < ng; c += (int64_t)gridDim.x * blockDim.x) {
    const int64_t b = c / gpr, cg = c - b * gpr;
    const T* base = in + b * a.R * a.K + cg * VEC;
    Acc acc[VEC];
#pragma unroll
    for (int q = 0; q < VEC; ++q) acc[q] = O::identity();
    int r = 0;
    for (; r + 3 < R; r += 4) {
      U128 x[4];
#pragma unroll
      for (int k = 0; k < 4; ++k) x[k] = ld_stream(base + (int64_t)(r + k) * a.K);
#pragma unroll
      for (int k = 0; k < 4; ++k)
#pragma unroll
        for (int q = 0; q < VEC; ++q) acc[q] = O::combine(acc[q], O::lift(unpack<T>(x[k], q)));
    }
    for (; r < R; ++r) {
      const U128 x = ld_stream(base + (int64_t)r * a.K);
#pragma unroll
      for (int q = 0; q < VEC; ++q) acc[q] = O::combine(acc[q], O::lift(unpack<T>(x, q)));
    }
    const int64_t o = b * a.K + cg * VEC;
#pragma unroll
    for (int q = 0; q < VEC; ++q) out[o + q] = merge_init<OP, T>(acc[q], out, o + q, a.init_from_out);
  }
}

// ------------------------------------------------------------- elementwise
template <int OP, typename T>
__global__ void __launch_bounds__(kBlock) ident_kernel(EltArgs a) {
  pdl_wait();  // no global access above this line
  pdl_trigger();
  using O = Op<OP, T>;
  const T* in = static_cast<const T*>(a.in);
  T* out = static_cast<T*>(a.out);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < a.n; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = merge_init<OP, T>(O::lift(in[i]), out, i, a.init_from_out);
}

template <int OP, typename T>
__global__ void __launch_bounds__(kBlock) fill_kernel(EltArgs a) {
  pdl_wait();  // no global access above this line
  pdl_trigger();
  using O = Op<OP, T>;
  T* out = static_cast<T*>(a.out);
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < a.n; i += (int64_t)gridDim.x * blockDim.x)
    out[i] = merge_init<OP, T>(O::identity(), out, i, a.init_from_out);
}

// Fixed rank-order combine of gathered partial results (sharded path).
template <int OP, typename T>
__global__ void __launch_bounds__(kBlock) gather_combine_kernel(const T* g, int nranks, int64_t n, T* out) {
  pdl_wait();  // no global access above this line
  pdl_trigger();
  using O = Op<OP, T>;
  for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    typename O::Acc v = O::identity();
    for (int r = 0; r < nranks; ++r) v = O::combine(v, O::lift(g[(int64_t)r * n + i]));
    out[i] = O::finish(v);
  }
}

// ------------------------------------------------------------- host launch
// Ring depth of the stream kernel (16 KiB stages); the planner sizes units
// for kStages.  XR_STREAM_NS=6 (A/B build): 96 KiB rings, 2 CTAs / SM.
#ifndef XR_STREAM_NS
#define XR_STREAM_NS 4
#endif

template <int OP, typename T>
cudaError_t launch_typed(Plan& p, int num_sms, cudaStream_t s) {
  constexpr int VEC = 16 / sizeof(T);
  switch (p.kernel) {
    case K_NONE:
      return cudaSuccess;
    case K_FILL: {
      const int64_t grid = grid_for((p.elt.n + kBlock - 1) / kBlock, num_sms, 8);
      if (cudaError_t e = launch_pdl(fill_kernel<OP, T>, dim3((unsigned)grid), dim3(kBlock), 0, s, p.elt)) return e;
      break;
    }
    case K_IDENT: {
      const int64_t grid = grid_for((p.elt.n + kBlock - 1) / kBlock, num_sms, 8);
      if (cudaError_t e = launch_pdl(ident_kernel<OP, T>, dim3((unsigned)grid), dim3(kBlock), 0, s, p.elt)) return e;
      break;
    }
    case K_SEG: {
      const int64_t groups_per_cta = kBlock / p.group;
      const int64_t ctas = (p.units + groups_per_cta - 1) / groups_per_cta;
      if (p.group == 8) {
        const int occ = occ_dev<seg_kernel<OP, T, 8, kBlock, kUnroll>>(kBlock, 0);
        if (cudaError_t e = launch_pdl(seg_kernel<OP, T, 8, kBlock, kUnroll>, dim3((unsigned)grid_for(ctas, num_sms, occ)), dim3(kBlock), 0, s, p.seg)) return e;
      } else if (p.group == 32) {
        const int occ = occ_dev<seg_kernel<OP, T, 32, kBlock, kUnroll>>(kBlock, 0);
        if (cudaError_t e = launch_pdl(seg_kernel<OP, T, 32, kBlock, kUnroll>, dim3((unsigned)grid_for(ctas, num_sms, occ)), dim3(kBlock), 0, s, p.seg)) return e;
      } else {
        const int occ = occ_dev<seg_kernel<OP, T, kBlock, kBlock, kUnroll>>(kBlock, 0);
        if (cudaError_t e = launch_pdl(seg_kernel<OP, T, kBlock, kBlock, kUnroll>, dim3((unsigned)grid_for(ctas, num_sms, occ)), dim3(kBlock), 0, s, p.seg)) return e;
      }
      break;
    }
    case K_STREAM: {
      auto kern = stream_kernel<OP, T, XR_STREAM_NS, kStageBytes>;
      constexpr int dyn = XR_STREAM_NS * kStageBytes;
      int occ = occ_dev<stream_kernel<OP, T, XR_STREAM_NS, kStageBytes>>(kWsEpiBlock, dyn);
      // Resident CTAs per SM by unit length: 3 for units < 128 KiB, else 2.
      // Short units must stream longer than a claim round trip (~1.5-2 us)
      // to hide it, so they want the slower per-CTA rate of 3 CTAs per SM
      // (r02au / r02av interleaved A/B: 512 MiB whole arrays, 64 KiB units,
      // 91.4 -> 81.2 us; 1 GiB fp64, 113 KiB units, 163.7 -> 155.4; 16-256 MiB
      // 3-10 % faster); long units keep 2 (2^30 fp32, 453 KiB units, 583.7 vs
      // 585.5; 32768^2 rows, 128 KiB units, 578.5 vs 582.0; 256 KiB KR units
      // level).  XR_STREAM_CTAS_PER_SM overrides.
      {
        const int64_t unit_bytes = p.seg.O * p.seg.C * p.seg.L * (int64_t)sizeof(T) / std::max<int64_t>(p.units, 1);
        const char* e = std::getenv("XR_STREAM_CTAS_PER_SM");
        occ = std::max(1, std::min(occ, e ? std::atoi(e) : unit_bytes < (int64_t(128) << 10) ? 3 : 2));
      }
      if (cudaError_t e = launch_pdl(kern, dim3((unsigned)grid_for(p.units, num_sms, occ)), dim3(kWsEpiBlock), dyn, s,
                                     p.seg))
        return e;
      break;
    }
    case K_RKR: {
      constexpr int dyn = kStages * kStageBytes;
      const bool narrow = p.rkr.L * (int64_t)sizeof(T) < 512;
      const int occ = narrow ? occ_dev<rkr_kernel<OP, T, kStages, true>>(kWsEpiBlock, dyn)
                             : occ_dev<rkr_kernel<OP, T, kStages, false>>(kWsEpiBlock, dyn);
      int64_t grid = grid_for(p.units, num_sms, occ);
      if (p.grid_hint > 0) grid = std::min(grid, p.grid_hint);
      if (cudaError_t e = narrow ? launch_pdl(rkr_kernel<OP, T, kStages, true>, dim3((unsigned)grid), dim3(kWsEpiBlock), dyn, s, p.rkr)
                                 : launch_pdl(rkr_kernel<OP, T, kStages, false>, dim3((unsigned)grid), dim3(kWsEpiBlock), dyn, s, p.rkr))
        return e;
      break;
    }
    case K_ROWS: {
      auto kern = rows_kernel<OP, T, kStages>;
      constexpr int dyn = kStages * kStageBytes;
      const int occ = occ_dev<rows_kernel<OP, T, kStages>>(kWsBlock, dyn);
      int64_t grid = grid_for(p.units, num_sms, occ);
      if (p.grid_hint > 0) grid = std::min(grid, p.grid_hint);
      if (cudaError_t e = launch_pdl(kern, dim3((unsigned)grid), dim3(kWsBlock), dyn, s, p.seg)) return e;
      break;
    }
    case K_RCLUSTER: {
      // one cluster of 16 CTAs (non-portable size; 8 if the device cannot
      // co-schedule 16), cluster dimension set at launch
      auto kern = rcluster_kernel<OP, T>;
      static int csize[kMaxDevices];  // 0 = not yet probed on that device
      int dev = 0;
      if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= kMaxDevices) { cudaGetLastError(); dev = 0; }
      int n = __atomic_load_n(&csize[dev], __ATOMIC_RELAXED);
      cudaLaunchConfig_t cfg = {};
      cfg.blockDim = dim3(kClusterBlock);
      cfg.stream = s;
      cudaLaunchAttribute attr[2];
      attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
      attr[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
      attr[1].id = cudaLaunchAttributeClusterDimension;
      cfg.attrs = attr;
      cfg.numAttrs = 2;
      if (n == 0) {
        n = 8;
        if (cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1) == cudaSuccess) {
          int active = 0;
          cfg.gridDim = dim3(kClusterCtas);
          attr[1].val.clusterDim.x = kClusterCtas;
          attr[1].val.clusterDim.y = 1;
          attr[1].val.clusterDim.z = 1;
          if (cudaOccupancyMaxActiveClusters(&active, kern, &cfg) == cudaSuccess && active > 0) n = kClusterCtas;
        }
        cudaGetLastError();
        __atomic_store_n(&csize[dev], n, __ATOMIC_RELAXED);
      }
      cfg.gridDim = dim3((unsigned)n);
      attr[1].val.clusterDim.x = (unsigned)n;
      attr[1].val.clusterDim.y = 1;
      attr[1].val.clusterDim.z = 1;
      if (cudaError_t e = cudaLaunchKernelEx(&cfg, kern, p.seg)) return e;
      break;
    }
    case K_THINCOL: {
      const int occ = occ_dev<thincol_kernel<OP, T>>(kBlock, 0);
      const int64_t ng = p.col.B * p.col.K / (16 / (int64_t)sizeof(T));
      if (cudaError_t e = launch_pdl(thincol_kernel<OP, T>, dim3((unsigned)grid_for((ng + kBlock - 1) / kBlock, num_sms, occ)), dim3(kBlock), 0, s, p.col)) return e;
      break;
    }
    case K_SHORTROW: {
      const int64_t row_bytes = p.seg.L * (int64_t)sizeof(T);
      const int64_t work = (p.seg.O * row_bytes + 63) / 64;  // 64-B chunks
      if (row_bytes > 64) {
        const int occ = occ_dev<shortrow_kernel<OP, T, 128>>(kBlock, 0);
        if (cudaError_t e = launch_pdl(shortrow_kernel<OP, T, 128>, dim3((unsigned)grid_for((work + 2 * kBlock - 1) / (2 * kBlock), num_sms, occ)), dim3(kBlock), 0, s, p.seg)) return e;
      } else {
        const int occ = occ_dev<shortrow_kernel<OP, T, 64>>(kBlock, 0);
        if (cudaError_t e = launch_pdl(shortrow_kernel<OP, T, 64>, dim3((unsigned)grid_for((work + kBlock - 1) / kBlock, num_sms, occ)), dim3(kBlock), 0, s, p.seg)) return e;
      }
      break;
    }
    case K_COLSMALL: {
      const int64_t grid = (p.units + kBlock / 32 - 1) / (kBlock / 32);
      if (cudaError_t e = launch_pdl(colsmall_kernel<OP, T>, dim3((unsigned)grid), dim3(kBlock), 0, s, p.col)) return e;
      break;
    }
    case K_COLFLAT: {
      const int occ = occ_dev<colflat_kernel<OP, T>>(kBlock, 0);
      if (cudaError_t e = launch_pdl(colflat_kernel<OP, T>, dim3((unsigned)grid_for(p.units, num_sms, occ)), dim3(kBlock), 0, s, p.col)) return e;
      break;
    }
    case K_COLTMA: {
      constexpr int dyn = kStages * kStageBytes;
      auto go = [&](auto kern, int occ) -> cudaError_t {
        int64_t grid = grid_for(p.units, num_sms, occ);
        if (p.grid_hint > 0) grid = std::min(grid, p.grid_hint);
        return launch_pdl(kern, dim3((unsigned)grid), dim3(kWsBlock), dyn, s, p.tmap, p.col);
      };
      cudaError_t e;
      if (p.col.box == 256) e = go(coltma_kernel<OP, T, kStages, 256>, occ_dev<coltma_kernel<OP, T, kStages, 256>>(kWsBlock, dyn));
      else if (p.col.box == 512) e = go(coltma_kernel<OP, T, kStages, 512>, occ_dev<coltma_kernel<OP, T, kStages, 512>>(kWsBlock, dyn));
      else e = go(coltma_kernel<OP, T, kStages, 1024>, occ_dev<coltma_kernel<OP, T, kStages, 1024>>(kWsBlock, dyn));
      if (e) return e;
      break;
    }
    case K_COL: {
      if (p.vec == VEC && VEC > 1) {
        const int occ = occ_dev<col_kernel<OP, T, VEC, kBlock, kUnroll>>(kBlock, 0);
        if (cudaError_t e = launch_pdl(col_kernel<OP, T, VEC, kBlock, kUnroll>, dim3((unsigned)grid_for(p.units, num_sms, occ)), dim3(kBlock), 0, s, p.col)) return e;
      } else {
        const int occ = occ_dev<col_kernel<OP, T, 1, kBlock, kUnroll>>(kBlock, 0);
        if (cudaError_t e = launch_pdl(col_kernel<OP, T, 1, kBlock, kUnroll>, dim3((unsigned)grid_for(p.units, num_sms, occ)), dim3(kBlock), 0, s, p.col)) return e;
      }
      break;
    }
    default:
      return cudaErrorInvalidValue;
  }
  count_launch();
  return cudaPeekAtLastError();
}

template <int OP, typename T>
cudaError_t launch_gather_typed(const void* g, int nranks, int64_t n, void* out, cudaStream_t s) {
  const int64_t grid = std::max<int64_t>(1, std::min<int64_t>((n + kBlock - 1) / kBlock, 148 * 8));
  if (cudaError_t e = launch_pdl(gather_combine_kernel<OP, T>, dim3((unsigned)grid), dim3(kBlock), 0, s,
                                 static_cast<const T*>(g), nranks, n, static_cast<T*>(out)))
    return e;
  count_launch();
  return cudaPeekAtLastError();
}

}  // namespace xr
