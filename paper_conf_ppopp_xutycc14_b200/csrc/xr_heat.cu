// xr_heat.cu -- config 4: the paper's 2-D heat equation application with its
// per-iteration max-residual reduction (section 4 @39322-41386,
// Fig 13(a) @43561-44280), fused into ONE kernel per sweep:
//
//   T2[j][i] = 0.25*((T1[j-1][i] + T1[j+1][i]) + (T1[j][i-1] + T1[j][i+1]))
//   residual = max(0, max_{j,i} |T1[j][i] - T2[j][i]|)       (reading C14)
//
// The paper runs the update and then a separate gang(+vector) max reduction
// that re-reads temp1/temp2 and copies `error` to the host every iteration
// (@40016-40410); fusing the residual into the sweep makes it free: 16 B per
// point per iteration (read T1 once from HBM, write T2 once; neighbours come
// from registers, shuffles and L1), and the reduction reuses the warp / CTA /
// last-CTA tiers of xr_ops.cuh.  Arithmetic uses __dadd_rn/__dmul_rn so no FMA
// contraction can occur (the paper disables FMA, @35389-35893), which makes
// the result bit-identical to the oracle.
#include <algorithm>
#include <cstdlib>
#include <utility>
#include <vector>

#include "../../include/xreduce.h"
#include "xr_internal.h"
#include "xr_ops.cuh"

namespace xr {

int heat_workspace(cudaStream_t s, int64_t pbytes, int64_t ntick, void** partials, unsigned** tickets);

constexpr int kHeatRows = 64;     // rows marched per warp (halo re-read: 2/64)
constexpr int kHeatPrefetch = 4;  // rows in flight per lane
constexpr int kHeatRowsPersistent = 12;  // output rows per tile of the persistent kernel

struct HeatArgs {
  const double* T1;
  double* T2;
  double* residual;
  double* partials;
  unsigned* tickets;
  int64_t nj, ni;
  int64_t jb, je;  // output rows [jb, je) of the buffer (single GPU: [1, nj-1))
  int64_t rows;    // output rows per CTA (bulk kernel: sized for one full wave)
  int64_t ntiles;  // CTAs in the grid
  const double* res_init;  // non-null: *residual = max(*res_init, this sweep's max) (split sweeps)
};

__device__ __forceinline__ double stencil(double up, double down, double left, double right) {
  return __dmul_rn(0.25, __dadd_rn(__dadd_rn(up, down), __dadd_rn(left, right)));
}

__device__ __forceinline__ double ld_row(const double* p) { return __ldg(p); }

// VEC = columns per lane (2: 16-B loads, needs ni even and 16-B aligned rows).
// Each warp marches down kHeatRows rows of a 32*VEC-column strip.  Rows are
// loaded PF rows ahead into a register ring (static indices via full unroll),
// so every lane keeps PF independent 16-B loads in flight: the sweep is an
// HBM stream, and one load per lane per row left it latency bound (68% of
// peak in profiles/ r01).
template <int VEC>
__global__ void __launch_bounds__(kBlock) heat_kernel(HeatArgs a) {
  pdl_wait();  // no global access above this line
  pdl_trigger();
  using O = Op<OP_MAX, double>;
  constexpr int NW = kBlock / 32;
  constexpr int STRIP = 32 * VEC;
  constexpr int PF = kHeatPrefetch;
  __shared__ double smem[32];
  __shared__ int s_last;
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int64_t c0 = ((int64_t)blockIdx.x * NW + warp) * STRIP;  // first column of my strip
  const int64_t col = c0 + (int64_t)lane * VEC;                   // my first column
  const int64_t j0 = a.jb + (int64_t)blockIdx.y * a.rows;
  const int64_t j1 = min(j0 + a.rows, a.je);
  const int64_t ni = a.ni;
  double err = 0.0;  // |d| >= 0, and the residual's initial value is 0 (C14)

  if (j0 < j1 && c0 < ni) {
    const bool have = col < ni;
    const double* base = a.T1 + col;
    // rows past j1 (the last one this warp needs) are never read
    auto load = [&](int64_t j, double (&v)[VEC]) {
      if (have && j <= j1) {
        if constexpr (VEC == 2) {
          const double2 x = __ldg(reinterpret_cast<const double2*>(base + j * ni));
          v[0] = x.x;
          v[1] = x.y;
        } else {
          v[0] = ld_row(base + j * ni);
        }
      } else {
#pragma unroll
        for (int q = 0; q < VEC; ++q) v[q] = 0.0;
      }
    };
    double up[VEC], cur[VEC], ring[PF][VEC];
    load(j0 - 1, up);
    load(j0, cur);
#pragma unroll
    for (int k = 0; k < PF; ++k) load(j0 + 1 + k, ring[k]);
    for (int64_t jb = j0; jb < j1; jb += PF) {
      double next[PF][VEC];
#pragma unroll
      for (int k = 0; k < PF; ++k) load(jb + 1 + PF + k, next[k]);  // next group in flight
#pragma unroll
      for (int k = 0; k < PF; ++k) {
        const int64_t j = jb + k;
        if (j < j1) {  // warp-uniform
          // left neighbour of my first column, right neighbour of my last column
          double left = __shfl_up_sync(0xffffffffu, cur[VEC - 1], 1);
          double right = __shfl_down_sync(0xffffffffu, cur[0], 1);
          if (lane == 0 && col >= 1 && have) left = ld_row(base + j * ni - 1);
          if (lane == 31 && col + VEC < ni) right = ld_row(base + j * ni + VEC);
#pragma unroll
          for (int q = 0; q < VEC; ++q) {
            const double l = q == 0 ? left : cur[q - 1];
            const double r = q == VEC - 1 ? right : cur[q + 1];
            const double nv = stencil(up[q], ring[k][q], l, r);
            const int64_t i = col + q;
            if (i >= 1 && i < ni - 1) {
              __stcs(a.T2 + j * ni + i, nv);
              err = O::combine(err, fabs(__dadd_rn(cur[q], -nv)));
            }
          }
#pragma unroll
          for (int q = 0; q < VEC; ++q) {
            up[q] = cur[q];
            cur[q] = ring[k][q];
          }
        }
      }
#pragma unroll
      for (int k = 0; k < PF; ++k)
#pragma unroll
        for (int q = 0; q < VEC; ++q) ring[k][q] = next[k][q];
    }
  }
  // a2 + a3: warp and CTA max, then a4: last CTA combines all CTA partials
  err = block_reduce<OP_MAX, double, kBlock>(err, smem);
  const int64_t cta = (int64_t)blockIdx.y * gridDim.x + blockIdx.x;
  if (threadIdx.x == 0) {
    a.partials[cta] = err;
    const unsigned t = ticket_add(a.tickets);
    s_last = (t == (unsigned)(a.ntiles - 1));
  }
  __syncthreads();
  if (s_last) {
    __threadfence();
    double w = 0.0;
    for (int64_t k = threadIdx.x; k < a.ntiles; k += kBlock) w = O::combine(w, ld_partial(a.partials + k));
    w = block_reduce<OP_MAX, double, kBlock>(w, smem);
    if (threadIdx.x == 0) {
      *a.residual = a.res_init ? O::combine(*a.res_init, w) : w;
      *a.tickets = 0u;
    }
  }
}

// Bulk-copy variant (ni even, T1/T2 16-B aligned): the CTA owns a tile of
// kTileCols columns x kHeatRows rows.  Thread 0 streams the T1 row windows
// [c0-2, c0+kTileCols+2) of rows j0-1 .. j1 into a ring of kHeatSlots
// shared-memory slots with cp.async.bulk (completion on per-slot mbarriers),
// kHeatSlots-2 rows ahead; each thread computes 2 columns of a row from the
// three slots (up / cur / down), stores them with 16-B streaming stores and
// folds |T2 - T1| into its private max.  Bytes in flight no longer depend on
// registers, and every T1 byte is read from HBM once per tile (halo rows and
// columns are ~3% extra).
constexpr int kTileCols = 2 * kConsThreads;    // 512 doubles = 4 KiB per row
constexpr int kSlotDoubles = kTileCols + 4;    // + 2-column halo on both sides
constexpr int kSlotDoublesP = kTileCols + 8;   // persistent kernel: + 2 lead + 1 shift, 16-B rows
constexpr int kHeatSlots = 8;

__global__ void __launch_bounds__(kWsBlock) heat_bulk_kernel(HeatArgs a) {
  using O = Op<OP_MAX, double>;
  __shared__ __align__(128) double slots[kHeatSlots][kSlotDoubles];
  __shared__ __align__(8) uint64_t full[kHeatSlots];
  __shared__ __align__(8) uint64_t empty[kHeatSlots];
  __shared__ double smem[32];
  __shared__ int s_last;
  const int tid0 = threadIdx.x, warp = tid0 >> 5, lane = tid0 & 31;
  const int64_t ni = a.ni;
  const int64_t c0 = (int64_t)blockIdx.x * kTileCols;
  const int64_t j0 = a.jb + (int64_t)blockIdx.y * a.rows;
  const int64_t j1 = min(j0 + a.rows, a.je);      // output rows [j0, j1)
  const int64_t nrows = j1 - j0 + 2;              // loaded rows j0-1 .. j1
  // window of every row: columns [ws, we) placed at slot offset ws - (c0 - 2)
  const int64_t ws = max(c0 - 2, (int64_t)0), we = min(c0 + kTileCols + 2, ni);
  const unsigned wbytes = (unsigned)((we - ws) * 8);
  const int64_t soff = ws - (c0 - 2);

  if (tid0 == 0) {
    for (int k = 0; k < kHeatSlots; ++k) {
      mbar_init(&full[k], 1);
      mbar_init(&empty[k], kConsWarps);
    }
    fence_mbar_init();
  }
  __syncthreads();
  pdl_wait();  // no global access above this line
  pdl_trigger();
  if (warp == 0) {
    // producer warp: row q of the tile into slot q % kHeatSlots once the
    // consumers released the row kHeatSlots earlier
    if (lane == 0 && j0 < j1) {
      for (int64_t q = 0; q < nrows; ++q) {
        const int slot = (int)(q % kHeatSlots);
        if (q >= kHeatSlots) mbar_wait(&empty[slot], (unsigned)(((q / kHeatSlots) - 1) & 1));
        mbar_expect_tx(&full[slot], wbytes);
        bulk_g2s(&slots[slot][soff], a.T1 + (j0 - 1 + q) * ni + ws, wbytes, &full[slot]);
      }
    }
    return;
  }
  const int tid = tid0 - 32, cw = warp - 1;
  double err = 0.0;
  if (j0 < j1) {
    mbar_wait(&full[0], 0);  // row j0-1
    mbar_wait(&full[1], 0);  // row j0
    const int64_t col = c0 + 2 * tid;  // my two columns: col, col+1
    const int li = 2 + 2 * tid;        // their slot index
    const bool i0 = col >= 1 && col <= ni - 2;          // interior columns
    const bool i1 = col + 1 >= 1 && col + 1 <= ni - 2;
    for (int64_t r = 1; r < nrows - 1; ++r) {  // output row j = j0 + r - 1
      const int64_t rd = r + 1;               // the "down" row
      mbar_wait(&full[rd % kHeatSlots], (unsigned)((rd / kHeatSlots) & 1));
      if (i0 || i1) {
        const double* up = slots[(r - 1) % kHeatSlots];
        const double* cur = slots[r % kHeatSlots];
        const double* dn = slots[rd % kHeatSlots];
        const double2 u2 = *reinterpret_cast<const double2*>(up + li);
        const double2 c2 = *reinterpret_cast<const double2*>(cur + li);
        const double2 d2 = *reinterpret_cast<const double2*>(dn + li);
        const double l = cur[li - 1], rr = cur[li + 2];
        const double n0 = stencil(u2.x, d2.x, l, c2.y);
        const double n1 = stencil(u2.y, d2.y, c2.x, rr);
        double* dst = a.T2 + (j0 + r - 1) * ni + col;
        if (i0 && i1) {
          __stcs(reinterpret_cast<double2*>(dst), make_double2(n0, n1));
        } else if (i0) {
          __stcs(dst, n0);
        } else {
          __stcs(dst + 1, n1);
        }
        if (i0) err = O::combine(err, fabs(__dadd_rn(c2.x, -n0)));
        if (i1) err = O::combine(err, fabs(__dadd_rn(c2.y, -n1)));
      }
      fence_proxy_async_smem();  // generic reads before the async refill
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[(r - 1) % kHeatSlots]);  // row r-1 is dead for this warp
    }
  }
  // a2 + a3: warp and consumer-wide max, then a4: last CTA combines all CTA partials
  err = cons_reduce<OP_MAX, double>(err, smem, cw, lane);
  const int64_t cta = (int64_t)blockIdx.y * gridDim.x + blockIdx.x;
  if (tid == 0) {
    a.partials[cta] = err;
    const unsigned t = ticket_add(a.tickets);
    s_last = (t == (unsigned)(a.ntiles - 1));
  }
  cons_sync();
  if (s_last) {
    __threadfence();
    double w = 0.0;
    for (int64_t k = tid; k < a.ntiles; k += kConsThreads) w = O::combine(w, ld_partial(a.partials + k));
    w = cons_reduce<OP_MAX, double>(w, smem, cw, lane);
    if (tid == 0) {
      *a.residual = a.res_init ? O::combine(*a.res_init, w) : w;
      *a.tickets = 0u;
    }
  }
}

// Persistent variant of the bulk sweep: grid = resident CTAs; the producer
// warp claims tiles (row-block-major, so the halo rows shared by vertically
// adjacent tiles are re-read from L2) from a device counter and streams their
// rows through the ring WITHOUT draining between tiles; consumers release
// every row slot exactly once (row r-1 after output row r, the last two rows
// at the end of a tile).  Removes wave quantisation (2048 tiles on ~740
// resident CTAs) and the per-CTA fill / drain of the one-tile version.  The
// max residual is exact, so the result does not depend on tile assignment.
struct HeatPArgs {
  HeatArgs h;
  int64_t gx, gy;               // column tiles, row blocks
  unsigned long long* sched;    // [2] tile counter + exit counter
};

template <bool ODD>  // ODD: ni odd, rows staged with a per-row 8-B shift
__global__ void __launch_bounds__(kWsBlock, ODD ? 4 : 1) heat_persistent_kernel(HeatPArgs pa) {
  using O = Op<OP_MAX, double>;
  constexpr int RING = 8;
  // Row layout: global column c of a row staged from element e0 = ws - sh
  // (sh = 1 when the window start is not 16-B aligned, odd ni) sits at index
  // c - c0 + 4 + sh; rows stay 16-B aligned for the bulk copies.
  __shared__ __align__(128) double slots[kHeatSlots][kSlotDoublesP];
  __shared__ __align__(8) uint64_t full[kHeatSlots];
  __shared__ __align__(8) uint64_t empty[kHeatSlots];
  __shared__ long long s_tiles[RING];
  __shared__ double smem[32];
  __shared__ int s_last;
  const HeatArgs& a = pa.h;
  const int tid0 = threadIdx.x, warp = tid0 >> 5, lane = tid0 & 31;
  const int64_t ni = a.ni, ntiles = pa.gx * pa.gy;
  auto tile_geom = [&](long long t, int64_t* c0, int64_t* j0, int64_t* j1) {
    const int64_t ty = t / pa.gx, tx = t - ty * pa.gx;  // row-block-major
    *c0 = tx * kTileCols;
    *j0 = a.jb + ty * a.rows;
    *j1 = min(*j0 + a.rows, a.je);
  };
  if (tid0 == 0) {
    for (int k = 0; k < kHeatSlots; ++k) {
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
      unsigned q = 0;  // global row counter (slot = q % kHeatSlots, phase = q / kHeatSlots)
      int seq = 0;
      long long t = claim_first(pa.sched);
      while (true) {
        const long long nt = claim_next(pa.sched);
        const int slot0 = (int)(q % kHeatSlots);
        s_tiles[seq & (RING - 1)] = t < ntiles ? t : -1;
        ++seq;
        if (t >= ntiles) {
          if (q >= kHeatSlots) mbar_wait(&empty[slot0], ((q / kHeatSlots) - 1) & 1u);
          mbar_arrive(&full[slot0]);
          break;
        }
        int64_t c0, j0, j1;
        tile_geom(t, &c0, &j0, &j1);
        const int64_t ws = max(c0 - 2, (int64_t)0), we = min(c0 + kTileCols + 2, ni);
        const int64_t soff = ws - (c0 - 2);
        const int64_t total = a.nj * ni;
        for (int64_t r = 0; r < j1 - j0 + 2; ++r, ++q) {  // rows j0-1 .. j1
          const int slot = (int)(q % kHeatSlots);
          const int64_t e = (j0 - 1 + r) * ni + ws;
          int64_t sh = 0, cnt = we - ws;
          if constexpr (ODD) {
            sh = e & 1;                                  // T1 is 16-B aligned
            cnt = (we - ws + sh + 1) & ~(int64_t)1;      // whole 16-B pairs
            // never past the buffer: the dropped element is then the last column
            // of the buffer's last row, which only serves as a (boundary) halo value
            if (e - sh + cnt > total) cnt -= 2;
          }
          const unsigned wbytes = (unsigned)(cnt * 8);
          if (q >= kHeatSlots) mbar_wait(&empty[slot], ((q / kHeatSlots) - 1) & 1u);
          mbar_expect_tx(&full[slot], wbytes);
          bulk_g2s(&slots[slot][soff + 2], a.T1 + e - sh, wbytes, &full[slot]);
        }
        t = nt;
      }
      sched_exit(pa.sched);
    }
    return;
  }
  // ---------------- consumer warps
  // Ring bookkeeping in 32-bit unsigned counters and per-tile invariants
  // hoisted out of the row loop: the r01 loop recomputed 64-bit signed
  // modulo / division / row-address products per row (163 warp instructions
  // per row, issue slots 85 % busy in ncu r02x -- the sweep was issue bound,
  // not memory bound).
  static_assert((kHeatSlots & (kHeatSlots - 1)) == 0, "ring slots: power of two");
  const int tid = tid0 - 32, cw = warp - 1;
  double err = 0.0;
  int seq = 0;
  unsigned q = 0;  // global row counter, as the producer's
  const int li = 4 + 2 * tid;
  while (true) {
    mbar_wait(&full[q % kHeatSlots], (q / kHeatSlots) & 1u);  // first row of the tile
    const long long t = s_tiles[seq & (RING - 1)];
    ++seq;
    if (t < 0) break;
    int64_t c0, j0, j1;
    tile_geom(t, &c0, &j0, &j1);
    const int nout = (int)(j1 - j0);  // output rows j0 .. j1-1 (loaded rows j0-1 .. j1)
    const unsigned qb = q;            // ring index of row j0-1
    mbar_wait(&full[(qb + 1) % kHeatSlots], ((qb + 1) / kHeatSlots) & 1u);
    constexpr bool odd = ODD;
    // ODD (ni odd): the rows alternate their 16-B phase.  On a row whose
    // flat index j*ni + c0 is odd the thread's column pair moves one column
    // left, so its flat index -- and hence its T2 address and its position
    // in the row's staged window -- is 16-B aligned: the centre pair loads
    // and the store are 16-B vectors on every row; only the up / down pairs
    // (the other phase) are two 8-B loads.  Tile t covers columns
    // [c0 - p, c0 + 512 - p) on a row of phase p, so every column still
    // belongs to exactly one tile.  The window start ws is even and ni odd,
    // so the phase of output row j -- the parity of j*ni + ws -- is j & 1.
    const int64_t colA = c0 + 2 * tid;
    const bool a0 = colA >= 1 && colA <= ni - 2, a1 = colA + 1 >= 1 && colA + 1 <= ni - 2;  // phase 0
    const bool b0 = colA - 1 >= 1 && colA - 1 <= ni - 2, b1 = colA >= 1 && colA <= ni - 2;  // phase 1
    double* dst = a.T2 + j0 * ni + colA;  // output row j0, column pair of phase 0
    for (int r = 1; r <= nout; ++r, dst += ni) {
      const unsigned qd = qb + (unsigned)r + 1u;
      mbar_wait(&full[qd % kHeatSlots], (qd / kHeatSlots) & 1u);
      const int p = odd ? (int)((j0 + r - 1) & 1) : 0;  // phase of output row j0 + r - 1
      const bool i0 = p ? b0 : a0, i1 = p ? b1 : a1;
      if (i0 || i1) {
        const double* up = slots[(qb + (unsigned)r - 1u) % kHeatSlots];
        const double* cur = slots[(qb + (unsigned)r) % kHeatSlots];
        const double* dn = slots[qd % kHeatSlots];
        double2 u2, c2, d2;
        double l, rr;
        if constexpr (!odd) {  // every row 16-B aligned: vector loads
          u2 = *reinterpret_cast<const double2*>(up + li);
          c2 = *reinterpret_cast<const double2*>(cur + li);
          d2 = *reinterpret_cast<const double2*>(dn + li);
          l = cur[li - 1];
          rr = cur[li + 2];
        } else {
          // centre: column c sits at c - c0 + 4 + p, i.e. li for the pair
          // (aligned); up / down rows have the other phase 1 - p: li + 1 - 2p
          const int so = li + 1 - 2 * p;
          c2 = *reinterpret_cast<const double2*>(cur + li);
          u2 = make_double2(up[so], up[so + 1]);
          d2 = make_double2(dn[so], dn[so + 1]);
          l = cur[li - 1];
          rr = cur[li + 2];
        }
        const double n0 = stencil(u2.x, d2.x, l, c2.y);
        const double n1 = stencil(u2.y, d2.y, c2.x, rr);
        double* d = dst - p;
        if (i0 && i1) {
          __stcs(reinterpret_cast<double2*>(d), make_double2(n0, n1));
        } else {
          if (i0) __stcs(d, n0);
          if (i1) __stcs(d + 1, n1);
        }
        // |T1 - T2| is +0 or positive (or NaN), and err starts at +0: on that
        // domain the reading-C7 max (Op<OP_MAX>::combine: bit-AND of equal
        // operands, a NaN operand ignored) IS fmax, without its +-0 handling
        // (r02ac SASS: 18 instructions per combine -> DSETP/SEL)
        if (i0) err = fmax(err, fabs(__dadd_rn(c2.x, -n0)));
        if (i1) err = fmax(err, fabs(__dadd_rn(c2.y, -n1)));
      }
      // Row r-1 is dead: every value loaded from it was consumed above (the
      // stencil's adds issue only once their shared-memory loads returned),
      // so the release-arrive on `empty` orders the producer's refill after
      // those reads without a per-row proxy fence (MEMBAR + FENCE.VIEW.ASYNC,
      // the loop's top stall in r02ac) -- the pattern of TMA load pipelines.
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[(qb + (unsigned)r - 1u) % kHeatSlots]);
    }
    __syncwarp();
    if (lane == 0) {  // the tile's last two rows
      mbar_arrive(&empty[(qb + (unsigned)nout) % kHeatSlots]);
      mbar_arrive(&empty[(qb + (unsigned)nout + 1u) % kHeatSlots]);
    }
    q = qb + (unsigned)nout + 2u;
  }
  err = cons_reduce<OP_MAX, double>(err, smem, cw, lane);
  if (tid == 0) {
    a.partials[blockIdx.x] = err;
    s_last = (ticket_add(a.tickets) == gridDim.x - 1u);
  }
  cons_sync();
  if (s_last) {
    __threadfence();
    double w = 0.0;
    for (int64_t k = tid; k < gridDim.x; k += kConsThreads) w = O::combine(w, ld_partial(a.partials + k));
    w = cons_reduce<OP_MAX, double>(w, smem, cw, lane);
    if (tid == 0) {
      *a.residual = a.res_init ? O::combine(*a.res_init, w) : w;
      *a.tickets = 0u;
    }
  }
}

// Sweep output rows [jb, je) of an nj x ni buffer (rows jb-1 and je are read).
static int heat_launch(int64_t nj, int64_t ni, int64_t jb, int64_t je, const double* T1, double* T2,
                       double* residual, cudaStream_t s, const double* res_init = nullptr) {
  const bool al16 = ((uintptr_t)T1 % 16 == 0) && ((uintptr_t)T2 % 16 == 0);
  const bool v2 = (ni % 2 == 0) && al16;
  // odd ni: only the persistent kernel stages rows with a per-row 8-B shift
  const bool odd_bulk = (ni % 2 == 1) && al16 && ni >= 5 && je > jb && std::getenv("XR_NO_BULK") == nullptr &&
                        std::getenv("XR_HEAT_ONE_TILE") == nullptr && std::getenv("XR_NO_ODD_BULK") == nullptr;
  const bool bulk = (v2 && ni >= 4 && std::getenv("XR_NO_BULK") == nullptr) || odd_bulk;
  const int strip = bulk ? kTileCols : 32 * (v2 ? 2 : 1) * (kBlock / 32);
  const int64_t gx = (ni + strip - 1) / strip;
  // 64-row tiles (one tile per CTA: 2048 CTAs at 8192^2; the persistent kernel
  // claims them dynamically).  Sizing row blocks for one full wave of resident
  // one-tile CTAs measured slower (0.79 vs 0.89 of peak, r01).
  // The persistent bulk kernel balances best with short tiles (r01 sweep at
  // 8192^2: 8 rows 0.908, 12 rows 0.929, 16 rows 0.918, 64 rows 0.869 of peak;
  // halo rows come from L2).
  const char* hr = std::getenv("XR_HEAT_ROWS");  // tuning override
  const bool persistent = bulk && std::getenv("XR_HEAT_ONE_TILE") == nullptr;
  // odd widths (shifted staging, 8-B consumer loads) prefer longer tiles: r01
  // sweep at 8191^2 / 11585^2: 12 rows 0.812 / 0.842, 24 rows 0.837 / 0.864
  constexpr int64_t kHeatRowsOdd = 24;
  const int64_t rows = hr ? std::max(4, std::atoi(hr))
                          : (odd_bulk ? kHeatRowsOdd : persistent ? kHeatRowsPersistent : kHeatRows);
  const int64_t gy = je > jb ? (je - jb + rows - 1) / rows : 1;
  if (gy > 65535) return XR_ERR_INVALID;
  HeatArgs a;
  a.rows = rows;
  a.T1 = T1; a.T2 = T2; a.residual = residual; a.nj = nj; a.ni = ni; a.ntiles = gx * gy;
  a.res_init = res_init;
  a.jb = jb; a.je = je;
  void* partials = nullptr;
  unsigned* tickets = nullptr;
  int st = heat_workspace(s, a.ntiles * (int64_t)sizeof(double), 6, &partials, &tickets);  // ticket + 2 x u64
  if (st) return st;
  a.partials = static_cast<double*>(partials);
  a.tickets = tickets;
  dim3 grid((unsigned)gx, (unsigned)gy);
  const char* hp = std::getenv("XR_HEAT_ONE_TILE");  // A/B: one tile per CTA
  cudaError_t le = cudaSuccess;
  if (bulk && hp == nullptr && je > jb) {
    auto occ_of = [](auto kern) {
      int n = 0;
      if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&n, kern, kWsBlock, 0) != cudaSuccess || n < 1) n = 1;
      return n;
    };
    static const int occ_even = occ_of(heat_persistent_kernel<false>);
    static const int occ_odd = occ_of(heat_persistent_kernel<true>);
    const bool odd = (ni % 2) != 0;
    const int occ = odd ? occ_odd : occ_even;
    int dev = 0, sms = 148;
    if (cudaGetDevice(&dev) == cudaSuccess) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    HeatPArgs pa;
    pa.h = a;
    pa.gx = gx;
    pa.gy = gy;
    pa.sched = reinterpret_cast<unsigned long long*>(tickets + 2);  // after the residual ticket (8-B aligned)
    int occ_use = occ;
    if (const char* e = std::getenv("XR_HEAT_CTAS_PER_SM")) occ_use = std::max(1, std::min(occ, std::atoi(e)));  // A/B
    const int64_t pgrid = std::min<int64_t>(gx * gy, (int64_t)sms * occ_use);
    if (odd) le = launch_pdl(heat_persistent_kernel<true>, dim3((unsigned)pgrid), dim3(kWsBlock), 0, s, pa);
    else le = launch_pdl(heat_persistent_kernel<false>, dim3((unsigned)pgrid), dim3(kWsBlock), 0, s, pa);
  } else if (bulk) le = launch_pdl(heat_bulk_kernel, grid, dim3(kWsBlock), 0, s, a);
  else if (v2) le = launch_pdl(heat_kernel<2>, grid, dim3(kBlock), 0, s, a);
  else le = launch_pdl(heat_kernel<1>, grid, dim3(kBlock), 0, s, a);
  count_launch();
  if (le != cudaSuccess || cudaPeekAtLastError() != cudaSuccess) { cudaGetLastError(); return XR_ERR_CUDA; }
  return XR_OK;
}

// Row layout of rank r's slab: local rows 0 .. n+1 hold global
// rows r*n-1 .. (r+1)*n; rows 0 and n+1 are halos (unused at the global
// boundary).  Output rows: the owned rows minus the global boundary rows.
int heat_slab_rows(int64_t n_local, int nranks, int rank, int64_t* jb, int64_t* je) {
  if (n_local < 1 || nranks < 1 || rank < 0 || rank >= nranks) return XR_ERR_INVALID;
  *jb = 1 + (rank == 0 ? 1 : 0);
  *je = n_local + 1 - (rank == nranks - 1 ? 1 : 0);
  return XR_OK;
}

int heat_step_rows(int64_t nj, int64_t ni, int64_t jb, int64_t je, const double* T1, double* T2,
                   double* residual, cudaStream_t s, const double* res_init) {
  return heat_launch(nj, ni, jb, je, T1, T2, residual, s, res_init);
}

}  // namespace xr

using namespace xr;

extern "C" int xr_heat_step(int64_t nj, int64_t ni, const double* T1, double* T2, double* residual,
                            xr_stream_t stream) {
  if (nj < 0 || ni < 0) return XR_ERR_INVALID;
  if (!residual) return XR_ERR_INVALID;
  if ((nj * ni > 0) && (!T1 || !T2)) return XR_ERR_INVALID;
  if (nj > 0 && ni > 0 && (nj > (INT64_MAX / 8) / ni)) return XR_ERR_INVALID;
  if (T1 == T2 && nj * ni > 0) return XR_ERR_INVALID;
  return heat_launch(nj, ni, 1, nj > 2 ? nj - 1 : 1, T1, T2, residual, (cudaStream_t)stream);
}

extern "C" int xr_heat_run_sharded_sim(int64_t n_local, int64_t ni, int64_t iters, int nranks,
                                       double* const* T1s, double* const* T2s, double* residuals,
                                       xr_stream_t stream) {
  if (n_local < 1 || ni < 0 || iters < 0 || nranks < 1 || !T1s || !T2s) return XR_ERR_INVALID;
  if (iters > 0 && !residuals) return XR_ERR_INVALID;
  cudaStream_t s = (cudaStream_t)stream;
  const int64_t nj = n_local + 2;
  const size_t row = (size_t)ni * sizeof(double);
  double* tmp = nullptr;
  if (cudaMallocAsync(&tmp, (size_t)nranks * sizeof(double), s) != cudaSuccess) { cudaGetLastError(); return XR_ERR_NOMEM; }
  std::vector<double*> a(T1s, T1s + nranks), b(T2s, T2s + nranks);
  int st = XR_OK;
  for (int64_t it = 0; it < iters && !st; ++it) {
    for (int r = 0; r < nranks && !st; ++r) {
      int64_t jb, je;
      heat_slab_rows(n_local, nranks, r, &jb, &je);
      st = heat_launch(nj, ni, jb, je, a[r], b[r], tmp + r, s);
    }
    // halo exchange of the new field (the NCCL path does grouped send/recv)
    for (int r = 0; r < nranks && !st; ++r) {
      if (r > 0 && cudaMemcpyAsync(b[r], b[r - 1] + n_local * ni, row, cudaMemcpyDeviceToDevice, s) != cudaSuccess)
        st = XR_ERR_CUDA;
      if (r < nranks - 1 && cudaMemcpyAsync(b[r] + (n_local + 1) * ni, b[r + 1] + ni, row, cudaMemcpyDeviceToDevice, s) != cudaSuccess)
        st = XR_ERR_CUDA;
    }
    if (!st && gather_f64(OP_MAX, tmp, nranks, 1, residuals + it, s) != cudaSuccess) st = XR_ERR_CUDA;
    std::swap(a, b);
  }
  cudaFreeAsync(tmp, s);
  return st;
}

extern "C" int xr_heat_run(int64_t nj, int64_t ni, int64_t iters, double* T1, double* T2,
                           double* residuals, xr_stream_t stream) {
  if (iters < 0 || (iters > 0 && !residuals)) return XR_ERR_INVALID;
  double* a = T1;
  double* b = T2;
  for (int64_t it = 0; it < iters; ++it) {
    int st = xr_heat_step(nj, ni, a, b, residuals + it, stream);
    if (st) return st;
    double* t = a; a = b; b = t;
  }
  return XR_OK;
}
