// xr_plan.cpp -- SURVEY.md 8(a) step a0: canonicalise (dims, level_mask) into
// one of R / KR / RK / KRK / RKR / K and pick the kernel, group width, splits
// and work units.  Pure host code (no CUDA calls), unit-tested on CPU through
// xr_plan_describe.
//
// Why canonicalise: the paper binds levels to hardware (gang = blockIdx.x,
// worker = threadIdx.y, vector = threadIdx.x; PAPER.md @11499-11699, 2.2), so
// "memory coalescing is impossible in worker and gang partial reduction"
// (@26577).  Here the API level is decoupled from the hardware tier: lanes
// always run along the contiguous dimension, so every shape is coalesced.
//  (1) drop every level of extent 1 (reducing or keeping one element is a
//      no-op), (2) merge adjacent levels of the same status (row-major
//      adjacent levels are one contiguous level), (3) the remaining pattern is
//      one of R, KR, RK, KRK, RKR, K.
#include <unistd.h>  // environ

#include <algorithm>
#include <cstdlib>
#include <cstring>

#include "../../include/xreduce.h"
#include "xr_internal.h"

namespace xr {

int dtype_size(int dtype) { return (dtype == XR_INT64 || dtype == XR_FP64) ? 8 : 4; }

int acc_size(int op, int dtype) {
  if (op == XR_OP_LAND || op == XR_OP_LOR) return 4;
  return dtype_size(dtype);
}

static int64_t cdiv(int64_t a, int64_t b) { return (a + b - 1) / b; }

// Tuning / A-B overrides (XR_*), read on every call so tests can flip them,
// but with ONE pass over the environment instead of a getenv scan per name
// (the planner runs on every launch; r01: ~1 us of host time per call).
namespace {
struct XrEnv {
  int n = 0;
  const char* kv[16];
  const char* get(const char* name) const {
    const size_t len = std::strlen(name);
    for (int i = 0; i < n; ++i)
      if (std::strncmp(kv[i], name, len) == 0 && kv[i][len] == '=') return kv[i] + len + 1;
    return nullptr;
  }
};
void scan_env(XrEnv* e) {
  for (char** p = environ; p && *p && e->n < 16; ++p)
    if ((*p)[0] == 'X' && (*p)[1] == 'R' && (*p)[2] == '_') e->kv[e->n++] = *p;
}
}  // namespace

int64_t grid_for(int64_t units, int num_sms, int ctas_per_sm) {
  int64_t cap = (int64_t)std::max(num_sms, 1) * std::max(ctas_per_sm, 1);
  return std::max<int64_t>(1, std::min(units, cap));
}

void make_plan(int op, int dtype, const int64_t dims[3], unsigned mask, uint64_t in_addr,
               int num_sms, Plan* p, bool seg_only, int64_t want_override, bool sub_cta, bool no_tma) {
  *p = Plan();
  XrEnv env;
  scan_env(&env);
  bool seg_only_small = false;
  const int size = dtype_size(dtype);
  const int vec = 16 / size;
  const int asz = acc_size(op, dtype);
  const bool chain_capped = (op == XR_OP_ADD && dtype == XR_FP32);
  const int64_t target_ctas = (int64_t)std::max(num_sms, 1) * kTargetCtasPerSm;

  int64_t count = 1;
  bool zero_reduced = false;
  for (int d = 0; d < 3; ++d) {
    const bool red = (mask >> d) & 1u;
    if (!red) count *= dims[d];
    else if (dims[d] == 0) zero_reduced = true;
  }
  p->out_count = count;
  if (count == 0) {  // a kept extent of 0: empty output (C17)
    p->shape = XR_SHAPE_NONE;
    p->kernel = K_NONE;
    return;
  }
  if (zero_reduced) {  // a reduced extent of 0: out = init (C17)
    p->shape = XR_SHAPE_FILL;
    p->kernel = K_FILL;
    p->cdims[0] = count;
    p->units = count;
    p->elt.n = count;
    return;
  }

  // (1) drop extent-1 levels, (2) merge adjacent levels of equal status
  int64_t run_n[3];
  bool run_red[3];
  int nr = 0;
  for (int d = 0; d < 3; ++d) {
    if (dims[d] == 1) continue;
    const bool red = (mask >> d) & 1u;
    if (nr > 0 && run_red[nr - 1] == red) {
      run_n[nr - 1] *= dims[d];
    } else {
      run_n[nr] = dims[d];
      run_red[nr] = red;
      ++nr;
    }
  }
  for (int r = 0; r < nr; ++r) p->cdims[r] = run_n[r];
  // Small inputs are latency bound, not bandwidth bound: the staged (bulk /
  // TMA ring) kernels would run on a few dozen CTAs, so below kSmallBytes the
  // register kernels, which spread one load round over many CTAs, are used.
  const char* sb = env.get("XR_SMALL_BYTES");  // test / tuning override
  const int64_t small = sb ? std::atoll(sb) : kSmallBytes;
  {
    int64_t total = 1;
    for (int d = 0; d < 3; ++d) total *= dims[d];
    if (total * size < small) seg_only_small = true;
  }

  // (3) the pattern
  if (nr == 0 || (nr == 1 && !run_red[0])) {  // K: every reduced extent is 1
    p->shape = XR_SHAPE_IDENT;
    p->kernel = K_IDENT;
    p->cdims[0] = count;
    p->units = count;
    p->elt.n = count;
    return;
  }

  const bool is_col = (nr == 2 && run_red[0]) || (nr == 3 && !run_red[0]);
  if (is_col) {
    // RK(R, K) or KRK(B, R, K): lanes own contiguous kept columns.
    int64_t B = 1, R, K;
    if (nr == 2) { R = run_n[0]; K = run_n[1]; p->shape = XR_SHAPE_RK; }
    else { B = run_n[0]; R = run_n[1]; K = run_n[2]; p->shape = XR_SHAPE_KRK; }
    const bool aligned = ((K * size) % 16 == 0) && (in_addr % 16 == 0);
    const int cv = aligned ? vec : 1;
    // Few reduced rows (R <= 32) and many kept 16-B column groups: an
    // elementwise-style pass, a thread per column group folding its R rows
    // (thincol_kernel, r02bk: R = 2 was 874 us on the tiled column kernels)
    if (!seg_only && aligned && R <= 32 && B * K / vec >= 65536 && env.get("XR_NO_THINCOL") == nullptr) {
      p->kernel = K_THINCOL;
      p->vec = vec;
      p->splits = 1;
      p->units = B * K / vec;
      p->group = 1;
      ColArgs& c = p->col;
      c.B = B; c.R = R; c.K = K; c.tiles = 1; c.S = 1; c.units = p->units;
      return;
    }
    // seg_only (the fused multi-input / multi-variable launches): always the
    // register column decomposition below (their col_unit, xr_colunit.cuh)
    // Small inputs with few reduced rows: one warp per 32 B of kept columns
    // (colsmall_kernel), no gang tier -- the latency-bound testsuite nest.
    {
      const int64_t cw = 2 * vec;
      const int64_t groups = B * cdiv(K, cw);
      if (!seg_only && seg_only_small && aligned && R <= 256 && groups >= 256 &&
          env.get("XR_NO_COLSMALL") == nullptr) {
        p->kernel = K_COLSMALL;
        p->vec = vec;
        p->splits = 1;
        p->units = groups;  // warps
        p->group = 32;
        ColArgs& c = p->col;
        c.B = B; c.R = R; c.K = K; c.tiles = cdiv(K, cw); c.S = 1; c.units = groups;
        return;
      }
    }
    // Narrow rows (power-of-two row_bytes in [16, 512] B, or up to 4 KiB for
    // small inputs): the flat column kernel streams whole rows contiguously.
    const int64_t row_bytes = K * size;
    const bool pow2 = (row_bytes & (row_bytes - 1)) == 0;
    const char* efm = env.get("XR_FLAT_MAX_ROW");  // A/B: widest row (bytes) for large inputs
    const int64_t flat_max = efm ? std::atoll(efm) : 512;
    // (r02: any multiple of 16 B -- rounds of whole rows -- and non-power-of-
    // two rows below 1 KiB, which the TMA column kernel does not take)
    const bool flat_width = row_bytes <= std::min<int64_t>(flat_max, 4096) || (seg_only_small && row_bytes <= 4096) ||
                            (!pow2 && row_bytes < 1024 && env.get("XR_NO_FLAT_NPOW2") == nullptr);
    // (r02: 8-B rows of two 32-bit columns too, when every batch starts 16-B
    // aligned -- a 16-B vector then holds two whole rows)
    const bool flat8 = row_bytes == 8 && size == 4 && in_addr % 16 == 0 && (B == 1 || (R * 8) % 16 == 0) &&
                       env.get("XR_NO_FLAT8") == nullptr;
    if (!seg_only && ((aligned && (pow2 || env.get("XR_NO_FLAT_NPOW2") == nullptr) && row_bytes >= 16 && flat_width) || flat8) &&
        env.get("XR_NO_FLAT") == nullptr) {
      const int64_t rp4k = 4096 / row_bytes;
      const int64_t nblk = cdiv(R, rp4k);                   // 4 KiB row blocks per batch
      const char* eu = env.get("XR_FLAT_UNITS_PER_CTA");  // tuning overrides
      const char* er = env.get("XR_FLAT_MIN_ROUNDS");
      // ~1 long unit per resident CTA: each unit's epilogue folds a K-wide
      // partial row, so long units win (r01 sweep: 256 units 4.7 TB/s, 4096
      // units 2.5 TB/s on the paper's 2^20 x 2 x 32 int32 gang case)
      const int64_t want = (eu ? std::max(1, std::atoi(eu)) : 1) * target_ctas;
      const int64_t min_rounds = er ? std::max(1, std::atoi(er)) : 16;
      int64_t S = std::max<int64_t>(1, cdiv(want, B));
      S = std::min<int64_t>(S, std::max<int64_t>(1, nblk / min_rounds));  // >= min_rounds 4 KiB rounds per unit
      if (chain_capped) S = std::max<int64_t>(S, cdiv(nblk, (int64_t)kChainCap * kUnroll));
      S = std::max<int64_t>(1, std::min<int64_t>(S, nblk));
      const int64_t G2 = cdiv(S, kGroupFold);
      p->kernel = K_COLFLAT;
      p->vec = vec;
      p->splits = S;
      p->units = B * S;
      p->group = kBlock;
      ColArgs& c = p->col;
      if (S > 1) {
        p->ws_bytes = B * (S + G2) * K * asz;
        p->tickets = B * (G2 + 1);
        // 32-bit integer '+': one packed (sum, count) word per output column
        // instead of partial rows and two ticket levels (xr_ops.cuh PackedAdd)
        if (op == XR_OP_ADD && dtype == XR_INT32 && env.get("XR_NO_PACKED") == nullptr) {
          p->ws_bytes = 0;
          p->tickets = 2 * B * K;
          c.packed = 1;
        }
      }
      c.B = B; c.R = R; c.K = K; c.tiles = 1; c.S = S; c.units = p->units; c.G2 = G2;
      return;
    }
    // TMA path: 16-B aligned rows of >= 1 KiB (one box row), R < 2^31, inputs
    // of >= 48 MiB (r02av: the register column kernel is 22-30 % faster at
    // 16-32 MiB, the TMA kernel 12-16 % faster from 64 MiB)
    // (an explicit XR_SMALL_BYTES below that also lowers it: the tests' way
    // of running the staged kernels on small, ragged shapes)
    const char* ecm = env.get("XR_COLTMA_MIN_BYTES");
    const int64_t coltma_min = ecm ? std::atoll(ecm) : sb ? std::min<int64_t>(small, int64_t(48) << 20)
                                                          : (int64_t(48) << 20);
    if (!seg_only && !seg_only_small && aligned && K * size >= 1024 && B * R * K * size >= coltma_min &&
        R < (int64_t(1) << 31) && K < (int64_t(1) << 31) &&
        B < (int64_t(1) << 31) && env.get("XR_NO_TMA") == nullptr && !no_tma) {
      // Balance (measured r01 sweeps): the producer warp keeps every CTA's ring
      // full, so few long units per CTA are best, but the unit count must be an
      // exact multiple of the CTAs launched (896 units on 444 CTAs left 8
      // stragglers for a third round).  k units per CTA, grid = units / k.
      const int64_t cap = (int64_t)std::max(num_sms, 1) * 3;  // resident CTAs (64 KiB ring each)
      const char* upc = env.get("XR_COLTMA_UNITS_PER_CTA");  // tuning override
      int64_t tiles = 0, k = 0, BR = 0, TWt = 0;
      // box = bx bytes x (16 KiB / bx) rows; a tile is bx bytes of columns
      auto splits_for = [&](int bx) {
        TWt = bx / size;
        BR = kStageBytes / bx;
        tiles = cdiv(K, TWt);
        const int64_t base = B * tiles;
        // measured (r01 sweeps): 2 units per CTA is best with few column tiles
        // (512^3 G/W/GW: 0.95/0.95/0.97 at 1 GiB); with many tiles (cfg3: 128)
        // ~512 KiB units (up to 16 per CTA) win (1.04 vs 1.02)
        const int64_t k_auto = base >= 64
            ? std::min<int64_t>(16, std::max<int64_t>(2, (B * R * K * size) / (cap << 19))) : 2;
        k = upc ? std::max(1, std::atoi(upc)) : k_auto;
        int64_t S;
        if (base >= k * cap) {
          S = 1;
        } else {
          S = std::max<int64_t>(1, (k * cap) / base);
          S = std::min<int64_t>(S, std::max<int64_t>(1, R / (kStages * BR)));  // >= kStages boxes per unit
        }
        if (chain_capped) S = std::max<int64_t>(S, cdiv(R, (int64_t)kChainCap * 8));
        return std::max<int64_t>(1, std::min<int64_t>(S, R));
      };
      // Box width (r02ac same-process interleaved A/B, tools/ab_env.py,
      // profiles/ab_box_r02ac.jsonl): 8-byte split tiles (S > 1, the 64-bit GW
      // cells) stream best in 256-B boxes (165.1 vs 170.8 us); every other
      // measured shape is best or level at 1 KiB (64-bit G +1.3-1.5 %,
      // 32-bit G / W and GW within 1 %, cfg3 columns +0.8-0.9 % with narrower
      // boxes).
      int box = (size == 8 && splits_for(1024) > 1) ? 256 : 1024;
      if (const char* eb = env.get("XR_COLTMA_BOX")) {  // A/B override
        const int v = std::atoi(eb);
        if (v == 256 || v == 512 || v == 1024) box = v;
      }
      if (K * size < box) box = 1024;  // (K * size >= 1024 here)
      const int64_t S = splits_for(box);
      p->kernel = K_COLTMA;
      p->vec = vec;
      p->splits = S;
      p->units = B * tiles * S;
      // S == 1 (many column tiles): all resident CTAs claim the tiles
      // dynamically (r02 grid sweep, 512^3 64-bit G / W: 444 CTAs 158 / 156
      // us vs 164 / 162 us at the k-units-per-CTA grid of 410); S > 1: k
      // units per CTA as before
      p->grid_hint = S == 1 ? std::min<int64_t>(cap, p->units)
                            : std::min<int64_t>(cap, cdiv(p->units, std::max<int64_t>(k, cdiv(p->units, cap))));
      if (const char* eg = env.get("XR_COLTMA_GRID")) p->grid_hint = std::max(1, std::atoi(eg));  // A/B
      p->group = kBlock;
      p->sched = true;
      // two-level gang tier: groups of gf unit partials, then the groups.  One
      // group (a single level) while S <= 64; beyond, groups of 16 (r02al
      // interleaved A/B: 32-bit GW, S = 444: 95.6 / 91.5 -> 93.8 / 88.7 us;
      // a second level for S = 55 cost the 64-bit GW +2.3 %)
      int gf = S <= kGroupFold ? kGroupFold : 16;
      if (const char* eg = env.get("XR_COLTMA_GROUP")) gf = std::max(2, std::atoi(eg));  // A/B
      const int64_t G2 = cdiv(S, gf);
      if (S > 1) {
        p->ws_bytes = B * tiles * (S + G2) * TWt * asz;
        p->tickets = B * tiles * (G2 + 1);
      }
      ColArgs& c = p->col;
      c.B = B; c.R = R; c.K = K; c.tiles = tiles; c.S = S; c.units = p->units; c.G2 = G2; c.box = box;
      // split-major unit ids (r02ah same-process A/B: cfg3 columns 613.7 ->
      // 597.8 us, cfg5 GW -0.6 to -1.7 %; S == 1 plans are unaffected)
      c.smaj = env.get("XR_COLTMA_TILE_MAJOR") == nullptr ? 1 : 0;
      c.gf = gf;
      return;
    }
    const int64_t TW = 32 * cv;
    const int64_t tiles = cdiv(K, TW);
    const int64_t NW = kBlock / 32;
    int64_t S = 1;
    const int64_t base = B * tiles;
    const int64_t want_col = (seg_only && want_override > 0) ? want_override : kUnitsPerCta * target_ctas;
    if (base < want_col) {
      S = cdiv(want_col, base);
      // >= 4 load rounds per warp: on small inputs a split's extra ticket round
      // costs more than its parallelism buys (cfg1 G/W: 4.0 us unsplit vs 5.4 us)
      S = std::min<int64_t>(S, std::max<int64_t>(1, R / (4 * NW * kUnroll)));
      S = std::min<int64_t>(S, 128);  // the last CTA of a tile folds S rows (8 warps x 4 loads)
    }
    if (chain_capped) S = std::max<int64_t>(S, cdiv(R, (int64_t)kChainCap * NW * kUnroll));
    S = std::max<int64_t>(1, std::min<int64_t>(S, R));
    p->kernel = K_COL;
    p->vec = cv;
    p->splits = S;
    p->units = B * tiles * S;
    p->group = kBlock;
    p->sched = true;
    if (S > 1) {
      p->ws_bytes = B * tiles * S * TW * asz;
      p->tickets = B * tiles;
    }
    ColArgs& c = p->col;
    c.B = B; c.R = R; c.K = K; c.tiles = tiles; c.S = S; c.units = p->units;
    return;
  }

  // seg: R(N) [O=1, C=1], KR(K, L) [C=1], RKR(R1, K, R2) [C=R1, rowStride=K*R2]
  int64_t O, C, L, rowStride, oStride;
  if (nr == 1) { O = 1; C = 1; L = run_n[0]; rowStride = 0; oStride = 0; p->shape = XR_SHAPE_R; }
  else if (nr == 2) { O = run_n[0]; C = 1; L = run_n[1]; rowStride = 0; oStride = L; p->shape = XR_SHAPE_KR; }
  else { O = run_n[1]; C = run_n[0]; L = run_n[2]; rowStride = O * L; oStride = L; p->shape = XR_SHAPE_RKR; }

  const int64_t row_bytes = L * size;
  // RKR with 2-4 KiB rows and at least as many reduced rows per output as
  // outputs (C >= O: few outputs, long strided columns of rows) run faster on
  // the register seg kernel's finer units than on the ring kernels (r02aq
  // interleaved A/B over 12 shapes: C >= O 3-8 % faster on seg, C <= O / 4
  // 2-6 % slower; 1 KiB and 512 B rows stay on rkr, 6-81 % faster there).
  const bool rkr_to_seg = nr == 3 && row_bytes >= 2048 && row_bytes <= 4096 && C >= O &&
                          env.get("XR_RKR_RING") == nullptr;
  // RKR with short rows (power-of-two row_bytes in [512 B, 2 KiB], 16-B
  // aligned, at least one full 16 KiB j-block): the rkr rows kernel -- units
  // are (block of J = 16 KiB / row_bytes outputs, range of k), each stage one
  // bulk copy of J contiguous rows, accumulated per warp in registers.
  // narrow rows (16-496 B, multiples of 16 B, r02): rkr_kernel's NARROW
  // consumers (4 fixed rows per thread per stage); the seg kernel read them
  // at 0.7-1.5 TB/s
  const bool rkr_narrow = row_bytes >= 16 && row_bytes < 512 && env.get("XR_NO_RKR_NARROW") == nullptr;
  if (!seg_only && !seg_only_small && !rkr_to_seg && nr == 3 && (rkr_narrow || row_bytes >= 512) && row_bytes <= 2048 &&
      ((row_bytes & (row_bytes - 1)) == 0 || (rkr_narrow && row_bytes % 16 == 0)) && in_addr % 16 == 0 &&
      O >= kStageBytes / row_bytes &&
      env.get("XR_NO_RKR") == nullptr && env.get("XR_NO_BULK") == nullptr) {
    const int64_t J = kStageBytes / row_bytes;
    const int64_t njb = cdiv(O, J);
    const int64_t cap = (int64_t)std::max(num_sms, 1) * 3;  // resident CTAs (64 KiB ring each)
    const char* eu = env.get("XR_RKR_UNITS_PER_CTA");   // tuning override
    // r01 sweeps (512^3 32-bit GV): 4-6 units per CTA 0.89, 8 0.87-0.91, 12 0.87, 16 0.81
    const int64_t k = eu ? std::max(1, std::atoi(eu)) : 4;
    // k units per resident CTA, each >= kStages stages (k values)
    int64_t S = std::max<int64_t>(1, std::min<int64_t>(cdiv(k * cap, njb), C / kStages));
    // fp32 '+': each lane accumulator folds vpl elements per k (chains <= kChainCap)
    // (narrow rows: one element per accumulator per k)
    if (chain_capped) S = std::max<int64_t>(S, cdiv(C * std::max<int64_t>(1, row_bytes >> 9), (int64_t)kChainCap));
    S = std::max<int64_t>(1, std::min<int64_t>(S, C));
    p->kernel = K_RKR;
    p->group = 32;
    p->vec = vec;
    p->splits = S;
    p->units = njb * S;
    p->sched = true;
    // 2 CTAs per SM (r02 grid sweep, 512^3 32-bit GV: 88.5 us at 222 / 296
    // CTAs vs 90.4-91.5 us at 444)
    // narrow rows: every resident CTA (r02bb A/B: 3 / SM 1-5 % faster; their
    // consumers run the per-output tier themselves, a unit end is costlier)
    const int64_t per_sm = row_bytes < 512 ? 3 : 2;
    p->grid_hint = std::min<int64_t>((int64_t)std::max(num_sms, 1) * per_sm, p->units);
    if (const char* eg = env.get("XR_RKR_GRID")) p->grid_hint = std::max(1, std::atoi(eg));  // A/B
    if (S > 1) {
      p->ws_bytes = O * S * asz;
      p->tickets = O;
    }
    RkrArgs& r = p->rkr;
    r.K = O; r.L = L; r.C = C; r.S = S; r.units = p->units;
    return;
  }
  // SHORT contiguous rows (KR, row_bytes a power of two in [4 B, 128 B],
  // 16-B aligned): a thread per 64 / 128-B chunk of whole rows (shortrow_kernel)
  if (!seg_only && nr == 2 && row_bytes <= 128 && (row_bytes & (row_bytes - 1)) == 0 && in_addr % 16 == 0 &&
      env.get("XR_NO_SHORTROW") == nullptr) {
    p->kernel = K_SHORTROW;
    p->group = 1;
    p->vec = vec;
    p->splits = 1;
    p->units = O;
    SegArgs& s = p->seg;
    s.O = O; s.C = 1; s.L = L; s.rowStride = 0; s.oStride = L;
    s.Sr = 1; s.Sc = 1; s.units = O;
    return;
  }
  // short contiguous rows (KR, row_bytes a power of two in [512 B, 2 KiB],
  // 16-B aligned): whole rows streamed in blocks of 16 KiB stages (rows_kernel)
  if (!seg_only && !seg_only_small && nr == 2 && row_bytes >= 512 && row_bytes <= 2048 &&
      (row_bytes & (row_bytes - 1)) == 0 &&
      in_addr % 16 == 0 && env.get("XR_NO_BULK") == nullptr) {
    const int64_t rps = kStageBytes / row_bytes;
    const int64_t nst = cdiv(O, rps);
    const int64_t cap = (int64_t)std::max(num_sms, 1) * 3;
    // many short units: a unit boundary costs the rows kernel nothing (no
    // epilogue, the producer streams across it), and short units balance the
    // tail (r01 sweep, 512^3 32-bit V: 2 units per CTA 0.91 of peak, 8 0.95,
    // 32 1.00)
    const char* eu = env.get("XR_ROWS_UNITS_PER_CTA");  // tuning override
    const int64_t k = eu ? std::max(1, std::atoi(eu)) : 32;
    const int64_t units = std::max<int64_t>(1, std::min<int64_t>(nst, k * cap));
    p->kernel = K_ROWS;
    p->group = 32;
    p->vec = vec;
    p->splits = 1;
    p->units = units;
    p->sched = true;
    // every resident CTA while each keeps >= 4 stages (its ring full): the r01
    // grid of units / k left 16-256 MiB inputs on 32-256 CTAs (r02av: 16 MiB
    // of 2 KiB rows 29 us vs 8.4 on the register kernel)
    p->grid_hint = std::min<int64_t>(cap, std::max<int64_t>(cdiv(units, k), cdiv(nst, 4)));
    if (const char* eg = env.get("XR_ROWS_GRID")) p->grid_hint = std::max(1, std::atoi(eg));  // A/B
    SegArgs& s = p->seg;
    s.O = O; s.C = 1; s.L = L; s.rowStride = 0; s.oStride = L;
    s.Sr = 1; s.Sc = units; s.units = units;
    return;
  }
  // small whole-array reductions: one thread-block cluster, gang tier through
  // distributed shared memory (rcluster_kernel) -- 256 KiB to 4 MiB.  OPT-IN
  // (XR_CLUSTER=1): measured SLOWER than the seg kernel's last-CTA ticket on
  // the 2 MiB testsuite nest (CUDA-graph replay 5.5 vs 4.0 us, r02h) -- 16
  // SMs cannot pull 2 MiB from L2 as fast as 128 CTAs on 128 SMs.
  if (!seg_only && nr == 1 && row_bytes >= (int64_t(256) << 10) && row_bytes <= (int64_t(4) << 20) &&
      env.get("XR_CLUSTER") != nullptr) {
    p->kernel = K_RCLUSTER;
    p->shape = XR_SHAPE_R;
    p->group = kClusterBlock;
    p->block = kClusterBlock;
    p->vec = vec;
    p->splits = kClusterCtas;
    p->units = kClusterCtas;
    p->grid_hint = kClusterCtas;
    SegArgs& s = p->seg;
    s.O = 1; s.C = 1; s.L = L; s.rowStride = 0; s.oStride = 0;
    s.Sr = 1; s.Sc = kClusterCtas; s.units = kClusterCtas;
    return;
  }
  // warp groups for rows up to 64 KiB (longer rows take the stream kernel):
  // r02bd interleaved A/B, 512 MiB of 8 KiB rows 168.8 -> 78.8 us (fp64 173.0
  // -> 78.8), 16 KiB rows 95.5 -> 79.0, 32 KiB rows 106.0 -> 54.0 (256 MiB)
  // against CTA-wide groups (r01 limit 4 KiB); one 256 MiB case of 16 KiB
  // rows was 6 % slower
  const char* ew = env.get("XR_SEG_W32_MAX");  // A/B: widest row (bytes) for warp groups
  const int64_t w32_max = ew ? std::atoll(ew) : 65536;
  // 8-lane groups for KR rows below 4 KiB (four rows per warp in flight):
  // r02bh / r02bi interleaved A/B, 512 MiB of 500 / 1000 / 2000 / 3000 B rows
  // 348 / 176 / 101 / 92 -> 123 / 95 / 84 / 85 us, the 2 MiB cfg1 v nest
  // (512 B rows) 1.96 -> 1.62 us per graph-replayed call; RKR segments and
  // 4 KiB rows stay on 32 lanes (16-38 % and 2 % slower on 8)
  const char* ew8 = env.get("XR_SEG_W8_MAX");  // A/B: widest row (bytes) for 8-lane groups
  const int64_t w8_max = ew8 ? std::atoll(ew8) : C == 1 ? 4095 : 128;
  int W = (seg_only && !sub_cta) ? kBlock : row_bytes <= w8_max ? 8 : row_bytes <= w32_max ? 32 : kBlock;
  auto resident_groups = [&](int w) { return target_ctas * (kBlock / w); };
  auto min_unit_elems = [&](int w) { return (int64_t)w * vec * kUnroll; };
  const int64_t work = C * L;  // elements per output
  // CTA-wide groups claim units dynamically: over-decompose for tail balance
  const int64_t want_units = (seg_only && want_override > 0) ? want_override * (kBlock / W)
                             : (W == kBlock ? kUnitsPerCta : 2) * resident_groups(W);
  int64_t S = 1;
  if (O < want_units) {
    S = cdiv(want_units, O);
    // register path: one unrolled load round per thread is enough (small,
    // latency-bound inputs get many CTAs); the stream path re-caps below
    S = std::min<int64_t>(S, std::max<int64_t>(1, work / min_unit_elems(W)));
  }
  // long contiguous rows (R, KR): the bulk-copy stream kernel; every unit must
  // cover at least kStages stages so the producer stays <= 3 units ahead
  const int64_t stage_elems = kStageBytes / size;
  // RKR with 16-B aligned rows of >= 4 KiB: the same kernel streams each
  // unit's rows (one bulk copy per row piece).  r01 sweep on 512^3 GV: 64-bit
  // (4 KiB rows) 0.95-1.01 of peak vs 0.66-0.95 for the seg kernel; 32-bit
  // (2 KiB rows) no better than seg (0.83-0.87 both), so those stay on seg.
  const char* rkr_min = env.get("XR_RKR_STREAM_MIN_ROW");  // tuning override (bytes)
  const bool rkr_stream = nr == 3 && !rkr_to_seg && row_bytes >= (rkr_min ? std::atoll(rkr_min) : 4096) &&
                          row_bytes % 16 == 0 && in_addr % 16 == 0 && env.get("XR_NO_RKR_STREAM") == nullptr;
  const bool stream = !seg_only && !seg_only_small && env.get("XR_NO_BULK") == nullptr &&
                      ((C == 1 && row_bytes >= (int64_t)kStages * kStageBytes) || rkr_stream);
  if (stream) {
    // several outputs: amortise the epilogue (RKR: 512 KiB units, r01 sweep)
    const int64_t min_stages = O == 1 ? kStages : C > 1 ? 8 * kStages : 4 * kStages;
    S = std::min<int64_t>(S, std::max<int64_t>(1, work / (min_stages * stage_elems)));
  }
  // fp32 '+': per-thread chains <= kChainCap (stream: 16 accumulators per thread)
  if (chain_capped) S = std::max<int64_t>(S, cdiv(work, (int64_t)kChainCap * W * vec * kUnroll));
  if (stream && env.get("XR_STREAM_SPLITS") != nullptr)  // tuning override
    S = std::max<int64_t>(1, std::atoll(env.get("XR_STREAM_SPLITS")));
  if (stream) W = kBlock;  // CTA-wide units, claimed dynamically
  if (S > 1 && W < 32) W = 32;  // the gang-tier ticket runs per warp or per CTA
  int64_t Sr, Sc;
  if (C >= S || (stream && C > 1)) { Sr = std::min(S, C); Sc = 1; }  // stream RKR units are whole rows
  else { Sr = C; Sc = std::min<int64_t>(cdiv(S, C), std::max<int64_t>(1, L / vec)); }
  S = Sr * Sc;

  p->kernel = stream ? K_STREAM : K_SEG;
  p->group = W;
  p->sched = (W == kBlock);
  p->vec = vec;
  p->splits = S;
  p->units = O * S;
  if (S > 1) {
    p->ws_bytes = O * S * asz;
    p->tickets = O;
    // seg, 32-bit integer '+': the packed gang tier (xr_ops.cuh PackedAdd)
    // keeps sum and count of an output in one 64-bit word, no partials
    if (!stream && !seg_only && op == XR_OP_ADD && dtype == XR_INT32 && env.get("XR_NO_PACKED") == nullptr) {
      p->ws_bytes = 0;
      p->tickets = 2 * O;
      p->seg.packed = 1;
    }
  }
  if (stream && O == 1) {  // unit partials + one CTA-exit ticket, also when S == 1
    p->ws_bytes = std::max<int64_t>(S, 1) * asz;
    p->tickets = 1;
  }
  SegArgs& s = p->seg;
  s.O = O; s.C = C; s.L = L; s.rowStride = rowStride; s.oStride = oStride;
  s.Sr = Sr; s.Sc = Sc; s.units = p->units;
  s.smaj = (stream && C > 1 && env.get("XR_STREAM_SPLIT_MAJOR") != nullptr) ? 1 : 0;  // A/B
  // CTA-wide seg units without splits (KR rows of 4-64 KiB): static
  // round-robin units, no claim round trip per unit (r02bc interleaved A/B:
  // 16 KiB rows 58.7 -> 50.4 us, 8 KiB rows -5.5 %; with splits and tickets
  // the dynamic claims stay, static was 12 % slower there)
  s.seg_static = (!stream && W == kBlock && S == 1 && p->units >= 4 * target_ctas) ? 1 : 0;
  if (const char* es = env.get("XR_SEG_STATIC")) s.seg_static = std::atoi(es) != 0 ? 1 : 0;  // A/B

  // Guided units for the whole-array stream (R shape): per-CTA timelines
  // (tools/timeline.py) showed the equal-unit tail -- the CTAs finish over
  // about one unit duration (4 us at 512 MiB, 10 us at 4 GiB).  The per-CTA
  // rate varies by up to 1.6x under full load, so a unit may only be as long
  // as the work still queued behind it can cover: phase 0 keeps the equal
  // units (u0 = L / S) for all but the last R = 2 G u0 elements; phase k then
  // hands out 2G units of u0 / 2^k (half the remaining work), so the queued
  // work stays two fair-share unit durations ahead of every claim, down to
  // two-stage units.  (A first version started at half the array in G units,
  // "factoring": a slow CTA's first unit outlasted the rest by 60 us, r02c.)
  // MEASURED NEUTRAL (r02d / perf3 A/B on one box: 512 MiB 84.4 vs 84.5 us,
  // 4 GiB 583-588 vs 582-588 us, back-to-back within 0.5 us): the tail
  // shrinks from 4-10 us to 1.3-1.7 us but the short units' per-unit cost
  // (claim round trip, consumer epilogue) gives it back, so equal units stay
  // the default; XR_GUIDED=1 selects this schedule.
  if (stream && O == 1 && C == 1 && env.get("XR_STREAM_SPLITS") == nullptr && env.get("XR_GUIDED") != nullptr) {
    Guided& gd = s.gd;
    const int64_t G = (int64_t)std::max(num_sms, 1) * 3;      // resident CTAs (64 KiB ring each)
    const char* gm = env.get("XR_GUIDED_MIN_BYTES");  // tuning override (default: two stages)
    const int64_t min_len = std::max<int64_t>(vec, (gm ? std::max(16ll, std::atoll(gm)) : 2ll * kStageBytes) / size);
    const int64_t u0 = std::max<int64_t>(min_len, cdiv(cdiv(L, std::max<int64_t>(Sc, 1)), vec) * vec);
    const int64_t bulk = L > 2 * G * u0 ? (L - 2 * G * u0) / vec * vec : 0;  // phase boundaries stay 16-B aligned
    int64_t rem = L - bulk, c = 0, u = 0;
    int k = 0;
    if (bulk > 0) {  // phase 0: equal units over the bulk of the array
      gd.u0[k] = 0; gd.c0[k] = 0; gd.len[k] = u0;
      u = cdiv(bulk, u0);
      c = bulk;
      ++k;
      // the last phase-0 unit may be short: phase 1 starts right after it
    }
    int64_t len = u0 / 2 / vec * vec;
    while (k < kMaxPhases - 1 && len >= 2 * min_len && rem > 0) {
      int64_t part = std::max<int64_t>(rem / 2 / vec * vec, len);
      if (part >= rem - min_len) part = rem;
      gd.u0[k] = u; gd.c0[k] = c; gd.len[k] = len;
      u += cdiv(part, len); c += part; rem -= part; ++k;
      len = len / 2 / vec * vec;
    }
    if (rem > 0) {
      gd.u0[k] = u; gd.c0[k] = c; gd.len[k] = min_len;
      u += cdiv(rem, min_len);
      c += rem;
      ++k;
    }
    gd.u0[k] = u; gd.c0[k] = L;
    gd.nph = k;
    s.Sr = 1; s.Sc = u; s.units = u;
    p->splits = u;
    p->units = u;
    p->ws_bytes = u * asz;
  }
}

}  // namespace xr
