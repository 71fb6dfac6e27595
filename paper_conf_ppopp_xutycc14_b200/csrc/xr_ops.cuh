// xr_ops.cuh -- library-internal device helpers (memory access, TMA / bulk
// copies, mbarriers, warp specialisation).  The operator traits and the
// reduction tiers live in the public include/xreduce_device.cuh.
#pragma once
#include <cstdlib>
#include "../../include/xreduce_device.cuh"

namespace xr {

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
// 16 B of partials, L2-coherent (ld.global.cg)
__device__ __forceinline__ U128 ld_partial16(const void* p) {
  U128 r;
  asm volatile("ld.global.cg.v4.u32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.w[0]), "=r"(r.w[1]), "=r"(r.w[2]), "=r"(r.w[3])
               : "l"(p));
  return r;
}
// q-th accumulator packed in a 16-B vector (4-B or 8-B accumulators)
template <typename A> __device__ __forceinline__ A acc_at(const U128& u, int q) {
  A a;
  if constexpr (sizeof(A) == 4) memcpy(&a, &u.w[q], 4);
  else { const uint32_t lohi[2] = {u.w[2 * q], u.w[2 * q + 1]}; memcpy(&a, lohi, 8); }
  return a;
}

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

__device__ __forceinline__ unsigned long long globaltimer_ns() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}

// Programmatic dependent launch (sm_90+): a kernel launched with the
// programmatic-stream-serialization attribute may start while the previous
// kernel on the stream drains; every thread waits here (griddepcontrol.wait:
// the previous grid completed and its memory is visible) before touching
// global memory, after the CTA's prologue (barrier init).  The trigger, issued
// AFTER the wait, lets the NEXT such launch be scheduled once every CTA of
// this grid has issued it; its CTAs take SM slots as this grid's CTAs exit and
// sit in their own wait.  (Triggering before the wait let a chain of graph-
// replayed launches cascade -- every grid launched at once, each waiting on
// its predecessor -- and made 2 MiB calls 0.8 us slower, r02e.)  Both are
// no-ops for ordinary launches.
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }

// Host: launch `kern` with the programmatic-stream-serialization attribute
// (every library kernel calls pdl_trigger / pdl_wait before its first global
// access), or plainly when XR_NO_PDL is set (A/B).
inline bool pdl_enabled() { return std::getenv("XR_NO_PDL") == nullptr; }
template <typename... KArgs, typename... Args>
cudaError_t launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t dyn, cudaStream_t s, Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = dyn;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = pdl_enabled() ? 1 : 0;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, kern, args...);
}

// Per-CTA timeline (profiling only, xr_debug_timeline): when the launch
// carries a buffer, one thread appends (cta, event, unit, %globaltimer)
// records: buf[0] = records written (atomic), buf[1] = capacity, then 2 words
// per record.  A null buffer costs one predicated branch per event.
enum TlEvent : unsigned { TL_START = 0, TL_UNIT = 1, TL_UNIT_DONE = 2, TL_CONS_END = 3, TL_FOLD = 4, TL_END = 5 };
__device__ __forceinline__ void tl_event(unsigned long long* tl, unsigned ev, long long unit) {
  if (tl == nullptr) return;
  const unsigned long long i = atomicAdd(tl, 1ull);
  if (i >= tl[1]) return;
  tl[2 + 2 * i] = ((unsigned long long)blockIdx.x << 40) | ((unsigned long long)ev << 32) |
                  (unsigned long long)(unsigned)unit;
  tl[3 + 2 * i] = globaltimer_ns();
}

// Resident CTAs per SM of kernel KERN at `block` threads and `dyn` bytes of
// dynamic shared memory, cached PER DEVICE: the dynamic-smem attribute binds
// to the current device's module, so a process that drives a second GPU sets
// it again there (a function-local static would set it on the first device
// only).  Setting the attribute twice is harmless, so the cache needs no lock.
constexpr int kMaxDevices = 64;
template <auto KERN>
int occ_dev(int block, int dyn) {
  static int cache[kMaxDevices];  // 0 = not yet computed on that device
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= kMaxDevices) { cudaGetLastError(); dev = -1; }
  if (dev >= 0) {
    const int v = __atomic_load_n(&cache[dev], __ATOMIC_RELAXED);
    if (v > 0) return v;
  }
  if (dyn > 48 * 1024) cudaFuncSetAttribute(KERN, cudaFuncAttributeMaxDynamicSharedMemorySize, dyn);
  int n = 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, KERN, block, dyn) != cudaSuccess || n < 1) {
    cudaGetLastError();
    n = 1;
  }
  if (dev >= 0) __atomic_store_n(&cache[dev], n, __ATOMIC_RELAXED);
  return n;
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
constexpr int kWsEpiBlock = kWsBlock + 32;   // + an epilogue warp (stream kernel)

// Order this thread's generic-proxy shared-memory accesses before later
// async-proxy (bulk copy / TMA) accesses to the same memory: a consumer
// executes it before releasing a ring stage that the producer will refill.
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
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

namespace xr {
// Dynamic unit claiming for CTA-wide work: thread 0 fetches the next unit
// index (prefetched one unit ahead into a parity slot) from a device counter;
// the last CTA to exit resets the counters for the next launch.
// Gang-tier ticket (a4): __threadfence() orders the partial(s) written before
// it (cumulatively: the CTA's writes ordered before by bar.sync) ahead of the
// increment; the last arriver fences again before reading the partials.
// XR_TICKET_ACQREL=1: one atom.add.acq_rel.gpu instead (measured neutral, r01
// A/B; the proven fence + atomic stays the default)
#ifndef XR_TICKET_ACQREL
#define XR_TICKET_ACQREL 0
#endif
// Packed gang tier for 32-bit integer '+' (exact and order-free mod 2^32):
// one 64-bit word per output carries the running sum in the high half and the
// arrival count in the low half, so ONE relaxed atomic both deposits a
// split's partial and takes its ticket -- no partial store, no fence, no
// reload of the partials by the last arriver (the sum is in the atomic's
// return value).  The count never carries into the sum (S < 2^32); the sum's
// carry out of bit 63 drops, which is the mod-2^32 wrap of the result.
template <int OP, typename T>
struct PackedAdd {
  static constexpr bool value = OP == OP_ADD && !IsFp<T>::value && sizeof(T) == 4;
};
// Returns true for the last of S arrivals, with the total in *sum; that
// arrival resets the word for the next launch.
__device__ __forceinline__ bool packed_add_arrive(unsigned long long* w, uint32_t v, int64_t S, uint32_t* sum) {
  const unsigned long long old = atomicAdd(w, ((unsigned long long)v << 32) | 1ull);
  if ((uint32_t)old != (uint32_t)(S - 1)) return false;
  *sum = (uint32_t)(old >> 32) + v;
  *w = 0ull;
  return true;
}

__device__ __forceinline__ unsigned ticket_add(unsigned* t) {
#if XR_TICKET_ACQREL
  unsigned v;
  asm volatile("atom.add.acq_rel.gpu.global.u32 %0, [%1], 1;" : "=r"(v) : "l"(t) : "memory");
  return v;
#else
  __threadfence();
  return atomicAdd(t, 1u);
#endif
}

// XR_STATIC_FIRST=1: every CTA's first unit is blockIdx.x (saves one claim
// round trip) -- measured neutral on streams and 8% SLOWER on 512^3 32-bit GW
// columns (r01 A/B), so the first unit is claimed like the others.
#ifndef XR_STATIC_FIRST
#define XR_STATIC_FIRST 0
#endif
#if XR_STATIC_FIRST
__device__ __forceinline__ long long claim_first(unsigned long long*) { return (long long)blockIdx.x; }
__device__ __forceinline__ long long claim_next(unsigned long long* c) {
  return (long long)gridDim.x + (long long)atomicAdd(c, 1ull);
}
#else
__device__ __forceinline__ long long claim_next(unsigned long long* c) { return (long long)atomicAdd(c, 1ull); }
__device__ __forceinline__ long long claim_first(unsigned long long* c) { return claim_next(c); }
#endif
__device__ __forceinline__ void sched_exit(unsigned long long* c) {
  if (threadIdx.x == 0) {
    __threadfence();
    const unsigned long long t = atomicAdd(c + 1, 1ull);
    if (t == (unsigned long long)gridDim.x - 1ull) {
      c[0] = 0ull;
      c[1] = 0ull;
    }
  }
}

}  // namespace xr
