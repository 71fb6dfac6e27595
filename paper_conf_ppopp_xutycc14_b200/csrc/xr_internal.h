// xr_internal.h -- host <-> device interface shared by the library's own
// translation units (never installed, never seen by the oracle).
#pragma once
#include <cstdint>
#include <cuda.h>
#include <cuda_runtime.h>

namespace xr {

constexpr int kBlock = 256;     // threads per CTA for every reduction kernel
constexpr int kUnroll = 4;      // independent 16-B loads in flight per thread
constexpr int kChainCap = 4096; // max sequential fp32 '+' chain per accumulator (C9)
constexpr int kTargetCtasPerSm = 8;  // 2048 threads/SM at 256 threads/CTA
constexpr int kUnitsPerCta = 8;      // dynamic units per resident CTA (tail balance)

enum Kernel : int { K_NONE = 0, K_FILL = 1, K_IDENT = 2, K_SEG = 3, K_COL = 4, K_STREAM = 5, K_COLTMA = 6, K_ROWS = 7, K_COLFLAT = 8, K_RKR = 9, K_COLSMALL = 10, K_RCLUSTER = 11, K_SHORTROW = 12, K_THINCOL = 13 };
constexpr int kClusterCtas = 16;  // rcluster_kernel: one thread-block cluster (non-portable size)
constexpr int kClusterBlock = 1024;

constexpr int kStages = 4;          // bulk-copy ring depth (stream kernel)
constexpr int64_t kSmallBytes = int64_t(16) << 20;  // below: register kernels (latency bound)
constexpr int kStageBytes = 16384;  // bytes per stage

// Fused cross-GPU exchange of a whole-nest result (stretch): the
// last CTA writes its rank's value into every peer's mailbox over NVLink
// (CUDA IPC peer pointers), publishes an epoch flag, waits for all ranks and
// combines the nranks values in rank order -- no separate collective launch.
// Mailbox (uint64 words): [2 parities][kMaxRanks] value slots, then
// [kMaxRanks] epoch flags.
constexpr int kMaxRanks = 8;
constexpr int kMailboxWords = 3 * kMaxRanks;
struct ExchArgs {
  unsigned long long* mine;                 // this rank's mailbox
  unsigned long long* peers[kMaxRanks];     // every rank's mailbox (peers[rank] == mine)
  int nranks, rank;
  unsigned long long epoch;                 // > 0, increments per call
  unsigned long long timeout_ns;            // bound on the wait for the peers (%globaltimer)
  int* status;                              // set to 1 if a peer never arrived within timeout_ns
                                            // (host-mapped: readable without a device sync)
};

// Guided unit schedule of the stream kernel's whole-array (R) shape (opt-in,
// XR_GUIDED=1; xr_plan.cpp has the measurements): phase k holds units
// [u0[k], u0[k+1]) of len[k] elements each, starting at element c0[k] (the
// last unit of a phase ends at c0[k+1]).  Phase 0 keeps the equal units, the
// later phases halve the unit length so the CTAs finish within about one
// short unit of each other.
constexpr int kMaxPhases = 12;
struct Guided {
  int nph;                       // 0: equal units (Sr x Sc split)
  int64_t u0[kMaxPhases + 1];
  int64_t c0[kMaxPhases + 1];
  int64_t len[kMaxPhases];
};

// Segmented rows ("seg"): out[o] = (+)_{r<C} (+)_{i<L} in[o*oStride + r*rowStride + i]
// -- covers R (O=1, C=1), KR (C=1) and RKR (C = outer reduced extent).
struct SegArgs {
  const void* in;
  void* out;
  void* partials;      // Acc[units] when splits > 1
  unsigned* tickets;   // [O] when splits > 1, zero between launches
  unsigned long long* sched;  // [2] dynamic unit counter + exit counter (CTA-wide groups)
  int64_t O, C, L, rowStride, oStride;
  int64_t Sr, Sc;      // splits over rows and over columns; S = Sr*Sc per output
  int64_t units;       // O * S
  int init_from_out;
  int packed;            // seg kernel, 32-bit int '+': packed (sum, count) gang tier, tickets = u64[O]
  int smaj;              // stream kernel, RKR: unit ids split-major (else output-major)
  int seg_static;        // seg kernel, CTA-wide units: static round-robin assignment (no claims)
  int use_exch;          // 1: fused exchange of the O == 1 result (exch below)
  ExchArgs exch;
  unsigned long long* tl;  // profiling timeline (xr_debug_timeline), null when off
  Guided gd;               // stream kernel, R shape: guided units (gd.nph > 0)
};

// Columns ("col"): out[b][c] = (+)_{r<R} in[b][r][c]  -- covers RK (B=1) and KRK.
struct ColArgs {
  const void* in;
  void* out;
  void* partials;      // Acc[B][tiles][S][32*vec] when S > 1
  unsigned* tickets;   // [B][tiles]
  unsigned long long* sched;  // [2] dynamic unit counter + exit counter
  int64_t B, R, K;
  int64_t tiles, S;
  int64_t units;       // B * tiles * S
  int64_t G2;          // coltma: groups of kGroupFold unit partials per tile (two-level gang tier)
  int box;             // coltma: TMA box width in bytes (256, 512 or 1024; tile = box columns)
  int packed;          // colflat, 32-bit int '+': packed (sum, count) gang tier, tickets = u64[B*K]
  int smaj;            // coltma: unit ids split-major (else tile-major)
  int gf;              // coltma: unit partials per group of the two-level gang tier
  int init_from_out;
  unsigned long long* tl;  // profiling timeline (coltma; xr_debug_timeline), null when off
};

#ifndef XR_GROUP_FOLD
#define XR_GROUP_FOLD 64
#endif
constexpr int kGroupFold = XR_GROUP_FOLD;  // unit partials folded per group by the group's last CTA

// Elementwise: out[o] = init (+) in[o] (ident) or out[o] = init (fill).
struct EltArgs {
  const void* in;
  void* out;
  int64_t n;
  int init_from_out;
};

// RKR rows kernel (xr_kernels.cuh rkr_kernel): out[j] = (+)_{k<C} (+)_{i<L}
// in[(k*K + j)*L + i]; units = (j-block of 16 KiB / row_bytes outputs, k split)
struct RkrArgs {
  const void* in;
  void* out;
  void* partials;          // Acc[K][S] when S > 1
  unsigned* tickets;       // [K] when S > 1, zero between launches
  unsigned long long* sched;
  int64_t K, L, C;         // outputs (middle extent), row length, outer reduced extent
  int64_t S, units;        // k splits per j-block, j-blocks * S
  int init_from_out;
};

struct Plan {
  int shape = 0;        // xr_shape
  int kernel = K_NONE;
  int64_t cdims[3] = {0, 0, 0};
  int64_t out_count = 0;
  int group = 0;        // seg group width
  int vec = 1;
  int64_t splits = 1;
  int64_t units = 0;
  int block = kBlock;
  int64_t ws_bytes = 0;
  int64_t tickets = 0;
  bool sched = false;   // CTA-wide units are claimed dynamically (2 extra counters)
  int64_t grid_hint = 0;  // >0: launch exactly this many CTAs (equal units per CTA)
  SegArgs seg{};
  ColArgs col{};
  CUtensorMap tmap{};   // K_COLTMA: 3-D map over (K, R, B), built at launch
  RkrArgs rkr{};
  EltArgs elt{};
};

// Pure host: validation happens before (api.cpp).  in_addr only matters for
// its alignment (16-B vector path of the column kernel).
// seg_only: plan for the register seg / column decompositions only, with
// CTA-wide groups (no stream / rows / TMA kernels) -- used by the fused
// transform-reduce and multi-variable launches.  want_units (> 0, seg_only
// only): the number of work units to aim for instead of the default
// over-decomposition (the multi-variable launch shares one grid among its
// variables), counted in CTA-wide units.  sub_cta (seg_only only): short rows
// keep the sub-CTA groups of 8 / 32 lanes (p->group) instead of CTA-wide ones.
// no_tma: never pick the TMA tensor-map column kernel (the launch re-plans
// with it when encoding the tensor map failed).
void make_plan(int op, int dtype, const int64_t dims[3], unsigned mask, uint64_t in_addr,
               int num_sms, Plan* p, bool seg_only = false, int64_t want_units = 0, bool sub_cta = false,
               bool no_tma = false);

int dtype_size(int dtype);
int acc_size(int op, int dtype);

// Launch the plan's kernel (exactly one launch unless kernel == K_NONE); the
// grid is min(units, num_sms * occupancy of the chosen kernel).
cudaError_t launch_i32(int op, Plan& p, int num_sms, cudaStream_t s);
cudaError_t launch_i64(int op, Plan& p, int num_sms, cudaStream_t s);
cudaError_t launch_f32(int op, Plan& p, int num_sms, cudaStream_t s);
cudaError_t launch_f64(int op, Plan& p, int num_sms, cudaStream_t s);

// Fixed rank-order combine of nranks gathered partial results (each `n`
// elements of dtype): out[i] = g[0][i] (+) g[1][i] (+) ... (sharded path).
cudaError_t gather_i32(int op, const void* g, int nranks, int64_t n, void* out, cudaStream_t s);
cudaError_t gather_i64(int op, const void* g, int nranks, int64_t n, void* out, cudaStream_t s);
cudaError_t gather_f32(int op, const void* g, int nranks, int64_t n, void* out, cudaStream_t s);
cudaError_t gather_f64(int op, const void* g, int nranks, int64_t n, void* out, cudaStream_t s);

// Encode the K_COLTMA tensor map for `in` (false if the driver entry point or
// the encode fails; the caller then re-plans with no_tma and launches the
// register column kernel instead).
bool make_col_tmap(CUtensorMap* m, int dtype, const void* in, int64_t B, int64_t R, int64_t K, int box_bytes);

// Grid for `units` work items given the device's resident-CTA budget.
int64_t grid_for(int64_t units, int num_sms, int ctas_per_sm);

void count_launch();

// The profiling timeline buffer set by xr_debug_timeline (null when off).
unsigned long long* debug_timeline();

}  // namespace xr
