// xr_api.cpp -- the C ABI (include/xreduce.h): validation, workspace, dispatch.
// Validation never touches CUDA, so every status path is testable on a CPU
// machine (tests/test_abi.py).
#include <algorithm>
#include <atomic>
#include <cstring>
#include <cstdlib>
#include <map>
#include <memory>
#include <mutex>
#include <utility>
#include <vector>

#include "../../include/xreduce.h"
#include "xr_internal.h"

namespace xr {

static std::atomic<int64_t> g_launches{0};
void count_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }
static std::atomic<unsigned long long*> g_timeline{nullptr};
unsigned long long* debug_timeline() { return g_timeline.load(std::memory_order_relaxed); }

static bool is_fp(int dtype) { return dtype == XR_FP32 || dtype == XR_FP64; }

// Argument validation shared by every entry point (no CUDA calls).
static int validate(int op, int dtype, const int64_t* dims, unsigned mask, int64_t* total,
                    int64_t* count) {
  if (op < XR_OP_ADD || op > XR_OP_LOR) return XR_ERR_INVALID;
  if (dtype < XR_INT32 || dtype > XR_FP64) return XR_ERR_INVALID;
  if (!dims) return XR_ERR_INVALID;
  if ((mask & 7u) == 0u || (mask & ~(7u | XR_INIT_FROM_OUT)) != 0u) return XR_ERR_INVALID;
  if (is_fp(dtype) && (op == XR_OP_BAND || op == XR_OP_BOR || op == XR_OP_BXOR))
    return XR_ERR_UNSUPPORTED;  // reading C3
  int64_t t = 1, c = 1;
  for (int d = 0; d < 3; ++d) {
    if (dims[d] < 0) return XR_ERR_INVALID;
    if (dims[d] != 0 && t > INT64_MAX / dims[d]) return XR_ERR_INVALID;
    t *= dims[d];
    if (!((mask >> d) & 1u)) c *= dims[d];
  }
  if (t > INT64_MAX / 8) return XR_ERR_INVALID;  // byte size must fit too
  *total = t;
  *count = c;
  return XR_OK;
}

static bool overlaps(const void* a, int64_t abytes, const void* b, int64_t bbytes) {
  if (abytes <= 0 || bbytes <= 0) return false;
  const uintptr_t a0 = (uintptr_t)a, b0 = (uintptr_t)b;
  return a0 < b0 + (uintptr_t)bbytes && b0 < a0 + (uintptr_t)abytes;
}

// Workspace per (device, stream): partials + zeroed tickets.  Tickets are
// reset by the last CTA of every launch; after a failed launch they are
// cleared again before the next use.
struct Workspace {
  void* partials = nullptr;
  size_t pbytes = 0;
  unsigned* tickets = nullptr;
  size_t ntickets = 0;
  bool dirty = false;
};
static std::mutex g_mu;
static std::map<std::pair<int, uintptr_t>, Workspace> g_ws;
static std::map<int, int> g_sms;

static int device_sms(int dev) {
  auto it = g_sms.find(dev);
  if (it != g_sms.end()) return it->second;
  int n = 0;
  if (cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess || n < 1) n = 148;
  g_sms[dev] = n;
  return n;
}

static int ensure_ws(Workspace& w, int64_t pbytes, int64_t ntick, cudaStream_t s) {
  if ((size_t)pbytes > w.pbytes || (size_t)ntick > w.ntickets) {
    // growth happens on the first calls only; wait for in-flight users
    if (w.partials || w.tickets) {
      if (cudaStreamSynchronize(s) != cudaSuccess) return XR_ERR_CUDA;
    }
    if ((size_t)pbytes > w.pbytes) {
      if (w.partials) cudaFree(w.partials);
      w.partials = nullptr;
      w.pbytes = 0;
      size_t want = ((size_t)pbytes * 5 / 4 + 4095) & ~(size_t)4095;
      if (cudaMalloc(&w.partials, want) != cudaSuccess) { cudaGetLastError(); return XR_ERR_NOMEM; }
      w.pbytes = want;
    }
    if ((size_t)ntick > w.ntickets) {
      if (w.tickets) cudaFree(w.tickets);
      w.tickets = nullptr;
      w.ntickets = 0;
      size_t want = ((size_t)ntick * 5 / 4 + 1023) & ~(size_t)1023;
      if (cudaMalloc(&w.tickets, want * sizeof(unsigned)) != cudaSuccess) { cudaGetLastError(); return XR_ERR_NOMEM; }
      w.ntickets = want;
      w.dirty = true;
    }
  }
  if (w.dirty && w.tickets) {
    if (cudaMemsetAsync(w.tickets, 0, w.ntickets * sizeof(unsigned), s) != cudaSuccess) return XR_ERR_CUDA;
    w.dirty = false;
  }
  return XR_OK;
}

static cudaError_t launch_dtype(int op, int dtype, Plan& p, int sms, cudaStream_t s) {
  switch (dtype) {
    case XR_INT32: return launch_i32(op, p, sms, s);
    case XR_INT64: return launch_i64(op, p, sms, s);
    case XR_FP32: return launch_f32(op, p, sms, s);
    default: return launch_f64(op, p, sms, s);
  }
}

static cudaError_t gather_dtype(int op, int dtype, const void* g, int nranks, int64_t n, void* out,
                                cudaStream_t s) {
  switch (dtype) {
    case XR_INT32: return gather_i32(op, g, nranks, n, out, s);
    case XR_INT64: return gather_i64(op, g, nranks, n, out, s);
    case XR_FP32: return gather_f32(op, g, nranks, n, out, s);
    default: return gather_f64(op, g, nranks, n, out, s);
  }
}

// Validated launch (caller holds no lock).  exch != nullptr: fused cross-GPU
// exchange of a whole-nest result (returns XR_ERR_UNSUPPORTED if the plan has
// no single-output CTA-wide tier to host it).
static int reduce_device(int op, int dtype, const int64_t* dims, unsigned mask, const void* in,
                         void* out, cudaStream_t stream, const ExchArgs* exch = nullptr) {
  int64_t total = 0, count = 0;
  int st = validate(op, dtype, dims, mask, &total, &count);
  if (st) return st;
  if (count == 0) return XR_OK;
  const int size = dtype_size(dtype);
  if (!out || (total > 0 && !in)) return XR_ERR_INVALID;
  if (((uintptr_t)out % size) || (total > 0 && ((uintptr_t)in % size))) return XR_ERR_INVALID;
  if (overlaps(in, total * size, out, count * size)) return XR_ERR_INVALID;

  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return XR_ERR_CUDA; }
  std::lock_guard<std::mutex> lock(g_mu);
  const int sms = device_sms(dev);
  Plan p;
  make_plan(op, dtype, dims, mask & 7u, (uint64_t)(uintptr_t)in, sms, &p);
  if (p.kernel == K_NONE) return XR_OK;
  if (exch && p.kernel == K_RCLUSTER)  // the fused exchange needs a CTA-wide last-CTA tier: seg plan
    make_plan(op, dtype, dims, mask & 7u, (uint64_t)(uintptr_t)in, sms, &p, /*seg_only=*/true);
  if (exch) {
    const bool ok = p.out_count == 1 &&
                    (p.kernel == K_STREAM || (p.kernel == K_SEG && p.group == kBlock));
    if (!ok) return XR_ERR_UNSUPPORTED;
    p.seg.use_exch = 1;
    p.seg.exch = *exch;
  }
  Workspace& w = g_ws[{dev, (uintptr_t)stream}];
  // tickets are followed by the two 64-bit scheduler counters (8-B aligned)
  const int64_t tick_words = (p.tickets + 1) & ~int64_t(1);
  st = ensure_ws(w, p.ws_bytes, tick_words + (p.sched ? 4 : 0), stream);
  if (st) return st;
  unsigned long long* sched = reinterpret_cast<unsigned long long*>(w.tickets + tick_words);
  p.seg.sched = sched;
  p.col.sched = sched;
  const int ifo = (mask & XR_INIT_FROM_OUT) ? 1 : 0;
  p.seg.in = in; p.seg.out = out; p.seg.partials = w.partials; p.seg.tickets = w.tickets;
  p.seg.init_from_out = ifo;
  p.seg.tl = debug_timeline();
  p.col.in = in; p.col.out = out; p.col.partials = w.partials; p.col.tickets = w.tickets;
  p.col.init_from_out = ifo;
  p.col.tl = debug_timeline();
  p.elt.in = in; p.elt.out = out; p.elt.init_from_out = ifo;
  p.rkr.in = in; p.rkr.out = out; p.rkr.partials = w.partials; p.rkr.tickets = w.tickets;
  p.rkr.sched = sched; p.rkr.init_from_out = ifo;
  if (p.kernel == K_COLTMA && !make_col_tmap(&p.tmap, dtype, in, p.col.B, p.col.R, p.col.K, p.col.box)) {
    // no tensor-map support (driver entry point or encode failed): re-plan
    // onto the register column kernels and launch those instead
    Plan q;
    make_plan(op, dtype, dims, mask & 7u, (uint64_t)(uintptr_t)in, sms, &q, false, 0, false, /*no_tma=*/true);
    q.seg = p.seg;  // keep the exchange fields (unused by column plans)
    p = q;
    const int64_t words = (p.tickets + 1) & ~int64_t(1);
    if ((st = ensure_ws(w, p.ws_bytes, words + (p.sched ? 4 : 0), stream))) return st;
    sched = reinterpret_cast<unsigned long long*>(w.tickets + words);
    p.col.in = in; p.col.out = out; p.col.partials = w.partials; p.col.tickets = w.tickets;
    p.col.init_from_out = ifo; p.col.sched = sched;
    p.elt.in = in; p.elt.out = out; p.elt.init_from_out = ifo;
  }
  cudaError_t e = launch_dtype(op, dtype, p, sms, stream);
  if (e != cudaSuccess) {
    cudaGetLastError();
    w.dirty = true;  // tickets may be left non-zero; clear before next use
    return XR_ERR_CUDA;
  }
  return XR_OK;
}

// ---------------------------------------------------------------- host-buffer path
// xr_reduce_host: the input is copied in bounded chunks through two device
// staging buffers on a copy stream, overlapping the H2D copy of chunk c+1 with
// the reduction of chunk c on the caller's stream (include/xreduce.h).  One
// staging context per (device, stream); the call is synchronous and holds the
// context's mutex throughout, so concurrent calls on different streams never
// share buffers and calls on one stream serialise.
constexpr size_t kHostChunkBytes = size_t(32) << 20;  // per staging buffer
struct Staging {
  std::mutex mu;
  void* in[2] = {nullptr, nullptr};
  size_t in_bytes = 0;
  void* out = nullptr;
  size_t out_bytes = 0;
  cudaStream_t copy = nullptr;
  cudaEvent_t copied[2] = {nullptr, nullptr};
  cudaEvent_t consumed[2] = {nullptr, nullptr};
};
static std::map<std::pair<int, uintptr_t>, std::unique_ptr<Staging>> g_stage;  // guarded by g_mu

static void free_staging(Staging& sg) {
  for (int b = 0; b < 2; ++b) {
    if (sg.in[b]) cudaFree(sg.in[b]);
    sg.in[b] = nullptr;
    if (sg.copied[b]) cudaEventDestroy(sg.copied[b]);
    if (sg.consumed[b]) cudaEventDestroy(sg.consumed[b]);
    sg.copied[b] = sg.consumed[b] = nullptr;
  }
  sg.in_bytes = 0;
  if (sg.out) cudaFree(sg.out);
  sg.out = nullptr;
  sg.out_bytes = 0;
  if (sg.copy) cudaStreamDestroy(sg.copy);
  sg.copy = nullptr;
}

// Buffers and streams for a call needing `chunk` bytes per input buffer and
// `obytes` of output (caller holds sg.mu; no work of this context is in flight).
static int prepare_staging(Staging& sg, size_t chunk, size_t obytes) {
  if (!sg.copy) {
    if (cudaStreamCreateWithFlags(&sg.copy, cudaStreamNonBlocking) != cudaSuccess) { cudaGetLastError(); return XR_ERR_CUDA; }
    for (int b = 0; b < 2; ++b)
      if (cudaEventCreateWithFlags(&sg.copied[b], cudaEventDisableTiming) != cudaSuccess ||
          cudaEventCreateWithFlags(&sg.consumed[b], cudaEventDisableTiming) != cudaSuccess) {
        cudaGetLastError();
        return XR_ERR_CUDA;
      }
  }
  if (chunk > sg.in_bytes) {
    for (int b = 0; b < 2; ++b) {
      if (sg.in[b]) cudaFree(sg.in[b]);
      sg.in[b] = nullptr;
    }
    sg.in_bytes = 0;
    for (int b = 0; b < 2; ++b)
      if (cudaMalloc(&sg.in[b], chunk) != cudaSuccess) { cudaGetLastError(); return XR_ERR_NOMEM; }
    sg.in_bytes = chunk;
  }
  if (obytes > sg.out_bytes) {
    if (sg.out) cudaFree(sg.out);
    sg.out = nullptr;
    sg.out_bytes = 0;
    if (cudaMalloc(&sg.out, obytes) != cudaSuccess) { cudaGetLastError(); return XR_ERR_NOMEM; }
    sg.out_bytes = obytes;
  }
  return XR_OK;
}

// One chunk of the nest: index prefix fixed on the levels before `lvl`, the
// range [a, a + ext) on level `lvl`, full extents after it.
struct HostChunk {
  int64_t dims[3];
  int64_t in_off;    // elements
  int64_t out_off;   // elements: the chunk's outputs are one contiguous block
  bool first;        // no earlier chunk wrote this output block
};

// Chunks of at most `cap` bytes in input order (exposed for the CPU tests
// through xr_host_chunks).  The chunk level is the outermost level whose
// single index fits in `cap`; a chunk's outputs are contiguous because every
// level after the chunk level is complete.  An output block is written first
// by the chunk whose indices on every REDUCED level up to the chunk level are
// 0; later chunks of the same block accumulate into it (init from out).
template <typename F>
static void for_each_chunk(const int64_t n[3], unsigned mask, int size, int64_t cap, F f) {
  int64_t row[3];  // bytes of one index of level d
  row[2] = size;
  row[1] = row[2] * n[2];
  row[0] = row[1] * n[1];
  int lvl = 2;
  for (int d = 0; d < 3; ++d)
    if (row[d] <= cap) { lvl = d; break; }
  const int64_t per = std::max<int64_t>(1, cap / row[lvl]);
  const int64_t istride[3] = {n[1] * n[2], n[2], 1};
  int64_t ostride[3];
  int64_t acc = 1;
  for (int d = 2; d >= 0; --d) {
    ostride[d] = acc;
    if (!((mask >> d) & 1u)) acc *= n[d];
  }
  const int64_t p0 = lvl > 0 ? n[0] : 1, p1 = lvl > 1 ? n[1] : 1;
  for (int64_t i0 = 0; i0 < p0; ++i0)
    for (int64_t i1 = 0; i1 < p1; ++i1)
      for (int64_t a = 0; a < n[lvl]; a += per) {
        HostChunk c;
        const int64_t idx[3] = {lvl == 0 ? a : i0, lvl == 1 ? a : (lvl > 1 ? i1 : 0), lvl == 2 ? a : 0};
        c.first = true;
        c.in_off = 0;
        c.out_off = 0;
        for (int d = 0; d < 3; ++d) {
          c.dims[d] = d < lvl ? 1 : d == lvl ? std::min(per, n[lvl] - a) : n[d];
          if (d > lvl) continue;
          c.in_off += idx[d] * istride[d];
          if ((mask >> d) & 1u) c.first = c.first && idx[d] == 0;
          else c.out_off += idx[d] * ostride[d];
        }
        f(c);
      }
}

static int64_t host_chunk_cap() {
  const char* e = std::getenv("XR_HOST_CHUNK_BYTES");  // test / tuning override
  const int64_t v = e ? std::atoll(e) : (int64_t)kHostChunkBytes;
  return std::max<int64_t>(v, 16);
}

static size_t chunk_bytes_for(int64_t total_bytes) {
  return (size_t)std::max<int64_t>(std::min<int64_t>(total_bytes, host_chunk_cap()), 16);
}

static int staging_for(xr_stream_t stream, Staging** out) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return XR_ERR_CUDA; }
  std::lock_guard<std::mutex> lock(g_mu);
  auto& slot = g_stage[{dev, (uintptr_t)stream}];
  if (!slot) slot.reset(new Staging());
  *out = slot.get();
  return XR_OK;
}

// The chunked H2D + reduce pipeline into the DEVICE output dout (which holds
// the init when mask has XR_INIT_FROM_OUT).  Caller holds sg.mu and has
// prepared the input buffers; enqueues only (the caller synchronises).
static int pipeline_locked(Staging& sg, int op, int dtype, const int64_t* dims, unsigned mask,
                           const void* in_host, char* dout, cudaStream_t s) {
  const int size = dtype_size(dtype);
  const int64_t total = dims[0] * dims[1] * dims[2];
  const bool ifo = (mask & XR_INIT_FROM_OUT) != 0;
  const unsigned base = mask & 7u;
  if (total == 0) return reduce_device(op, dtype, dims, mask, nullptr, dout, s);  // out = init (C17)
  // the copy stream starts after the caller's prior work on `stream`, and
  // never overwrites a buffer before the reduction reading it (chunk c-2)
  if (cudaEventRecord(sg.consumed[0], s) != cudaSuccess || cudaStreamWaitEvent(sg.copy, sg.consumed[0], 0) != cudaSuccess) {
    cudaGetLastError();
    return XR_ERR_CUDA;
  }
  int st = XR_OK;
  int64_t c = 0;
  for_each_chunk(dims, base, size, host_chunk_cap(), [&](const HostChunk& ch) {
    if (st) return;
    const int b = (int)(c & 1);
    const int64_t bytes = ch.dims[0] * ch.dims[1] * ch.dims[2] * size;
    if ((c >= 2 && cudaStreamWaitEvent(sg.copy, sg.consumed[b], 0) != cudaSuccess) ||
        cudaMemcpyAsync(sg.in[b], static_cast<const char*>(in_host) + ch.in_off * size, (size_t)bytes,
                        cudaMemcpyHostToDevice, sg.copy) != cudaSuccess ||
        cudaEventRecord(sg.copied[b], sg.copy) != cudaSuccess || cudaStreamWaitEvent(s, sg.copied[b], 0) != cudaSuccess) {
      cudaGetLastError();
      st = XR_ERR_CUDA;
      return;
    }
    const unsigned m = base | ((!ch.first || ifo) ? XR_INIT_FROM_OUT : 0u);
    st = reduce_device(op, dtype, ch.dims, m, sg.in[b], dout + ch.out_off * size, s);
    if (!st && cudaEventRecord(sg.consumed[b], s) != cudaSuccess) { cudaGetLastError(); st = XR_ERR_CUDA; }
    ++c;
  });
  return st;
}

// used by xr_comm.cpp (xr_reduce_sharded_host): the pipeline into a caller's
// device buffer; synchronous.
int reduce_host_into(int op, int dtype, const int64_t* dims, unsigned mask, const void* in_host, void* out_dev,
                     cudaStream_t s) {
  int64_t total = 0, count = 0;
  int st = validate(op, dtype, dims, mask, &total, &count);
  if (st) return st;
  if (count == 0) return XR_OK;
  if (!out_dev || (total > 0 && !in_host)) return XR_ERR_INVALID;
  Staging* sgp = nullptr;
  if ((st = staging_for((xr_stream_t)s, &sgp))) return st;
  Staging& sg = *sgp;
  std::lock_guard<std::mutex> call_lock(sg.mu);
  if ((st = prepare_staging(sg, chunk_bytes_for(total * dtype_size(dtype)), 0))) return st;
  st = pipeline_locked(sg, op, dtype, dims, mask, in_host, static_cast<char*>(out_dev), s);
  const cudaError_t e1 = cudaStreamSynchronize(sg.copy);
  const cudaError_t e2 = cudaStreamSynchronize(s);
  if (!st && (e1 != cudaSuccess || e2 != cudaSuccess)) st = XR_ERR_CUDA;
  if (st) cudaGetLastError();
  return st;
}

}  // namespace xr

using namespace xr;

extern "C" int xr_host_chunks(const int64_t nest_dims[3], unsigned level_mask, int dtype, int64_t cap_bytes,
                              int64_t max_chunks, int64_t* out6, int64_t* nchunks) {
  int64_t total = 0, count = 0;
  int st = validate(XR_OP_ADD, dtype, nest_dims, level_mask, &total, &count);
  if (st) return st;
  if (!nchunks || cap_bytes < 1 || max_chunks < 0 || (max_chunks > 0 && !out6)) return XR_ERR_INVALID;
  int64_t k = 0;
  if (total > 0)
    for_each_chunk(nest_dims, level_mask & 7u, dtype_size(dtype), cap_bytes, [&](const HostChunk& c) {
      if (k < max_chunks) {
        int64_t* o = out6 + 6 * k;
        o[0] = c.dims[0]; o[1] = c.dims[1]; o[2] = c.dims[2];
        o[3] = c.in_off; o[4] = c.out_off; o[5] = c.first ? 1 : 0;
      }
      ++k;
    });
  *nchunks = k;
  return XR_OK;
}

extern "C" {

int xr_reduce(int op, int dtype, const int64_t nest_dims[3], unsigned level_mask, const void* in,
              void* out, xr_stream_t stream) {
  return reduce_device(op, dtype, nest_dims, level_mask, in, out, (cudaStream_t)stream);
}

int xr_out_count(const int64_t nest_dims[3], unsigned level_mask, int64_t* count) {
  int64_t total = 0, c = 0;
  int st = validate(XR_OP_ADD, XR_INT32, nest_dims, level_mask, &total, &c);
  if (st) return st;
  if (!count) return XR_ERR_INVALID;
  *count = c;
  return XR_OK;
}

const char* xr_strerror(int status) {
  switch (status) {
    case XR_OK: return "XR_OK: success";
    case XR_ERR_INVALID: return "XR_ERR_INVALID: invalid argument";
    case XR_ERR_UNSUPPORTED: return "XR_ERR_UNSUPPORTED: operator not defined for this dtype";
    case XR_ERR_CUDA: return "XR_ERR_CUDA: CUDA runtime error";
    case XR_ERR_NCCL: return "XR_ERR_NCCL: NCCL error";
    case XR_ERR_NOMEM: return "XR_ERR_NOMEM: device allocation failed";
    default: return "unknown xreduce status";
  }
}

int xr_plan_describe(int op, int dtype, const int64_t nest_dims[3], unsigned level_mask,
                     uint64_t in_addr, int num_sms, xr_plan_info* info) {
  int64_t total = 0, count = 0;
  int st = validate(op, dtype, nest_dims, level_mask, &total, &count);
  if (st) return st;
  if (!info || num_sms < 1) return XR_ERR_INVALID;
  Plan p;
  make_plan(op, dtype, nest_dims, level_mask & 7u, in_addr, num_sms, &p);
  std::memset(info, 0, sizeof *info);
  info->shape = p.shape;
  info->kernel = p.kernel;
  for (int d = 0; d < 3; ++d) info->cdims[d] = p.cdims[d];
  info->out_count = p.out_count;
  info->group = p.group;
  info->vec = p.vec;
  info->splits = p.splits;
  info->units = p.units;
  info->block = p.block;
  int64_t ctas = p.units;
  if (p.kernel == K_COLTMA || p.kernel == K_ROWS || p.kernel == K_RKR) ctas = std::min<int64_t>(p.units, (int64_t)num_sms * 3);
  if (p.kernel == K_STREAM) ctas = std::min<int64_t>(p.units, (int64_t)num_sms * 2);  // 2 resident per SM
  if (p.kernel == K_SEG && p.group < p.block) ctas = (p.units + p.block / p.group - 1) / (p.block / p.group);
  if (p.kernel == K_FILL || p.kernel == K_IDENT) ctas = (p.units + kBlock - 1) / kBlock;
  if (p.kernel == K_COLSMALL) ctas = (p.units + kBlock / 32 - 1) / (kBlock / 32);
  info->grid = p.kernel == K_NONE ? 0 : grid_for(ctas, num_sms, kTargetCtasPerSm);
  if (p.grid_hint > 0) info->grid = std::min(info->grid, p.grid_hint);
  info->ws_bytes = p.ws_bytes;
  info->tickets = p.tickets;
  return XR_OK;
}

int xr_reserve(int op, int dtype, const int64_t nest_dims[3], unsigned level_mask, xr_stream_t stream) {
  int64_t total = 0, count = 0;
  int st = validate(op, dtype, nest_dims, level_mask, &total, &count);
  if (st) return st;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return XR_ERR_CUDA; }
  std::lock_guard<std::mutex> lock(g_mu);
  Plan p;
  // worst case over alignments: the column kernel's unaligned variant has more tiles
  make_plan(op, dtype, nest_dims, level_mask & 7u, 0, device_sms(dev), &p);
  Plan q;
  make_plan(op, dtype, nest_dims, level_mask & 7u, 4, device_sms(dev), &q);
  Workspace& w = g_ws[{dev, (uintptr_t)stream}];
  const int64_t words = std::max((p.tickets + 1) & ~int64_t(1), (q.tickets + 1) & ~int64_t(1)) + 4;
  return ensure_ws(w, std::max(p.ws_bytes, q.ws_bytes), words, (cudaStream_t)stream);
}

int xr_shutdown(void) {
  std::lock_guard<std::mutex> lock(g_mu);
  cudaDeviceSynchronize();
  for (auto& kv : g_ws) {
    if (kv.second.partials) cudaFree(kv.second.partials);
    if (kv.second.tickets) cudaFree(kv.second.tickets);
  }
  g_ws.clear();
  for (auto& kv : g_stage) {
    std::lock_guard<std::mutex> sl(kv.second->mu);
    free_staging(*kv.second);
  }
  g_stage.clear();
  cudaGetLastError();
  return XR_OK;
}

int64_t xr_launch_count(void) { return g_launches.load(); }

int xr_debug_timeline(void* buf, int64_t cap_records) {
  if (buf && cap_records < 1) return XR_ERR_INVALID;
  g_timeline.store(static_cast<unsigned long long*>(buf), std::memory_order_relaxed);
  return XR_OK;
}

int xr_reduce_host(int op, int dtype, const int64_t nest_dims[3], unsigned level_mask,
                   const void* in_host, void* out_host, xr_stream_t stream) {
  int64_t total = 0, count = 0;
  int st = validate(op, dtype, nest_dims, level_mask, &total, &count);
  if (st) return st;
  if (count == 0) return XR_OK;
  if (!out_host || (total > 0 && !in_host)) return XR_ERR_INVALID;
  const int size = dtype_size(dtype);
  cudaStream_t s = (cudaStream_t)stream;
  Staging* sgp = nullptr;
  if ((st = staging_for(stream, &sgp))) return st;
  Staging& sg = *sgp;
  std::lock_guard<std::mutex> call_lock(sg.mu);  // held for the whole (synchronous) call
  if ((st = prepare_staging(sg, chunk_bytes_for(total * size), (size_t)count * size))) return st;
  char* dout = static_cast<char*>(sg.out);
  if ((level_mask & XR_INIT_FROM_OUT) &&
      cudaMemcpyAsync(dout, out_host, (size_t)count * size, cudaMemcpyHostToDevice, s) != cudaSuccess) {
    cudaGetLastError();
    return XR_ERR_CUDA;
  }
  st = pipeline_locked(sg, op, dtype, nest_dims, level_mask, in_host, dout, s);
  if (!st && cudaMemcpyAsync(out_host, dout, (size_t)count * size, cudaMemcpyDeviceToHost, s) != cudaSuccess) {
    cudaGetLastError();
    st = XR_ERR_CUDA;
  }
  // both streams drain before the buffers can be reused (also on errors)
  const cudaError_t e1 = cudaStreamSynchronize(sg.copy);
  const cudaError_t e2 = cudaStreamSynchronize(s);
  if (!st && (e1 != cudaSuccess || e2 != cudaSuccess)) st = XR_ERR_CUDA;
  if (st) cudaGetLastError();
  return st;
}

// ------------------------------------------------------------ sharding plan
int xr_shard_plan(int op, int dtype, const int64_t local_dims[3], unsigned level_mask, int nranks,
                  int rank, xr_shard_info* info) {
  int64_t total = 0, count = 0;
  int st = validate(op, dtype, local_dims, level_mask, &total, &count);
  if (st) return st;
  if (!info || nranks < 1 || rank < 0 || rank >= nranks) return XR_ERR_INVALID;
  std::memset(info, 0, sizeof *info);
  const bool ifo = (level_mask & XR_INIT_FROM_OUT) != 0;
  info->local_count = count;
  info->gang_offset = (int64_t)rank * local_dims[0];
  if (level_mask & XR_GANG) {
    info->global_count = count;
    info->out_offset = 0;
    info->merge_init = (ifo && rank == 0) ? 1 : 0;  // merged exactly once
    info->local_init_from_out = info->merge_init;
    switch (op) {
      case XR_OP_ADD: info->collective = XR_COLL_ALLREDUCE; info->nccl_op = 0; break;  // ncclSum
      case XR_OP_MUL: info->collective = XR_COLL_ALLREDUCE; info->nccl_op = 1; break;  // ncclProd
      case XR_OP_MAX: info->collective = XR_COLL_ALLREDUCE; info->nccl_op = 2; break;  // ncclMax
      case XR_OP_MIN: info->collective = XR_COLL_ALLREDUCE; info->nccl_op = 3; break;  // ncclMin
      case XR_OP_LAND: info->collective = XR_COLL_ALLREDUCE; info->nccl_op = 3; break; // min of 0/1
      case XR_OP_LOR: info->collective = XR_COLL_ALLREDUCE; info->nccl_op = 2; break;  // max of 0/1
      default: info->collective = XR_COLL_ALLGATHER_COMBINE; info->nccl_op = -1; break;  // & | ^
    }
  } else {
    info->collective = XR_COLL_ALLGATHER;
    info->nccl_op = -1;
    info->global_count = count * nranks;
    info->out_offset = (int64_t)rank * count;
    info->merge_init = ifo ? 1 : 0;  // each rank merges its own segment's init
    info->local_init_from_out = info->merge_init;
  }
  if (count == 0) info->collective = XR_COLL_NONE;
  return XR_OK;
}

int xr_reduce_sharded_sim(int op, int dtype, const int64_t local_dims[3], unsigned level_mask,
                          const void* const* shards, int nranks, void* out, xr_stream_t stream) {
  int64_t total = 0, count = 0;
  int st = validate(op, dtype, local_dims, level_mask, &total, &count);
  if (st) return st;
  if (nranks < 1 || !shards) return XR_ERR_INVALID;
  if (count == 0) return XR_OK;
  if (!out) return XR_ERR_INVALID;
  const int size = dtype_size(dtype);
  cudaStream_t s = (cudaStream_t)stream;
  xr_shard_info info;
  if ((st = xr_shard_plan(op, dtype, local_dims, level_mask, nranks, 0, &info))) return st;
  const unsigned base_mask = level_mask & 7u;
  if (info.collective == XR_COLL_ALLGATHER) {
    for (int r = 0; r < nranks; ++r) {
      xr_shard_info ir;
      xr_shard_plan(op, dtype, local_dims, level_mask, nranks, r, &ir);
      char* seg = (char*)out + ir.out_offset * size;
      st = reduce_device(op, dtype, local_dims, base_mask | (ir.local_init_from_out ? XR_INIT_FROM_OUT : 0u),
                         shards[r], seg, s);
      if (st) return st;
    }
    return XR_OK;
  }
  // G in mask: every rank's partial into a gathered buffer, then the fixed
  // rank-order combine (the same kernel the NCCL path uses for & | ^).
  void* g = nullptr;
  if (cudaMallocAsync(&g, (size_t)nranks * count * size, s) != cudaSuccess) { cudaGetLastError(); return XR_ERR_NOMEM; }
  for (int r = 0; r < nranks && !st; ++r) {
    xr_shard_info ir;
    xr_shard_plan(op, dtype, local_dims, level_mask, nranks, r, &ir);
    char* dst = (char*)g + (size_t)r * count * size;
    if (ir.local_init_from_out &&
        cudaMemcpyAsync(dst, out, (size_t)count * size, cudaMemcpyDeviceToDevice, s) != cudaSuccess) {
      st = XR_ERR_CUDA;
      break;
    }
    st = reduce_device(op, dtype, local_dims, base_mask | (ir.local_init_from_out ? XR_INIT_FROM_OUT : 0u),
                       shards[r], dst, s);
  }
  if (!st && gather_dtype(op, dtype, g, nranks, count, out, s) != cudaSuccess) st = XR_ERR_CUDA;
  cudaFreeAsync(g, s);
  return st;
}

int xr_reduce_fused_sim(int op, int dtype, const int64_t local_dims[3], unsigned level_mask,
                        const void* const* shards, int nranks, void* const* outs) {
  int64_t total = 0, count = 0;
  int st = validate(op, dtype, local_dims, level_mask, &total, &count);
  if (st) return st;
  if (nranks < 1 || nranks > kMaxRanks || !shards || !outs || !(level_mask & XR_GANG) || count != 1)
    return XR_ERR_INVALID;
  const size_t mb_bytes = kMailboxWords * sizeof(unsigned long long);
  unsigned long long* mb = nullptr;
  int* status = nullptr;
  if (cudaMalloc(&mb, mb_bytes * nranks) != cudaSuccess || cudaMalloc(&status, sizeof(int)) != cudaSuccess) {
    cudaGetLastError();
    return XR_ERR_NOMEM;
  }
  cudaMemset(mb, 0, mb_bytes * nranks);
  cudaMemset(status, 0, sizeof(int));
  std::vector<cudaStream_t> ss(nranks);
  for (int r = 0; r < nranks; ++r) cudaStreamCreateWithFlags(&ss[r], cudaStreamNonBlocking);
  // warm-up per stream (workspace growth, lazy module loading): both may
  // synchronise the device, which must not happen while a rank's last CTA
  // spins waiting for the others
  unsigned long long saved = 0;  // rank 0's initial value survives the warm-up
  cudaMemcpy(&saved, outs[0], dtype_size(dtype), cudaMemcpyDeviceToHost);
  for (int r = 0; r < nranks && !st; ++r)
    st = reduce_device(op, dtype, local_dims, level_mask & 7u, shards[r], outs[r], ss[r]);
  cudaDeviceSynchronize();
  cudaMemcpy(outs[0], &saved, dtype_size(dtype), cudaMemcpyHostToDevice);
  // every "rank" is a concurrent kernel on its own stream; the last CTA of
  // each spins on its mailbox until all the others published (real protocol).
  // XR_TEST_SIM_SKIP_RANK=r (tests): rank r never launches, so the others
  // must time out (XR_EXCH_TIMEOUT_MS), leave their out unchanged and report.
  const char* skip_env = std::getenv("XR_TEST_SIM_SKIP_RANK");
  const int skip = skip_env ? std::atoi(skip_env) : -1;
  const char* to_env = std::getenv("XR_EXCH_TIMEOUT_MS");
  const unsigned long long timeout_ns =
      (unsigned long long)std::max(1ll, to_env ? std::atoll(to_env) : 10000ll) * 1000000ull;
  for (int r = 0; r < nranks && !st; ++r) {
    if (r == skip) continue;
    ExchArgs x{};
    x.mine = mb + (size_t)r * kMailboxWords;
    for (int p = 0; p < nranks; ++p) x.peers[p] = mb + (size_t)p * kMailboxWords;
    x.nranks = nranks;
    x.rank = r;
    x.epoch = 1;
    x.timeout_ns = timeout_ns;
    x.status = status;
    xr_shard_info info;
    xr_shard_plan(op, dtype, local_dims, level_mask, nranks, r, &info);
    const unsigned m = (level_mask & 7u) | (info.local_init_from_out ? XR_INIT_FROM_OUT : 0u);
    st = reduce_device(op, dtype, local_dims, m, shards[r], outs[r], ss[r], &x);
  }
  cudaDeviceSynchronize();
  int h_status = 0;
  cudaMemcpy(&h_status, status, sizeof(int), cudaMemcpyDeviceToHost);
  for (int r = 0; r < nranks; ++r) cudaStreamDestroy(ss[r]);
  cudaFree(mb);
  cudaFree(status);
  if (cudaGetLastError() != cudaSuccess) return XR_ERR_CUDA;
  if (!st && h_status) st = XR_ERR_NCCL;  // a rank never arrived
  return st;
}

}  // extern "C"

namespace xr {
// used by xr_comm.cpp
int reduce_device_checked(int op, int dtype, const int64_t* dims, unsigned mask, const void* in, void* out,
                          cudaStream_t s, const ExchArgs* exch) {
  return reduce_device(op, dtype, dims, mask, in, out, s, exch);
}
cudaError_t gather_combine(int op, int dtype, const void* g, int nranks, int64_t n, void* out, cudaStream_t s) {
  return gather_dtype(op, dtype, g, nranks, n, out, s);
}
// used by xr_xform.cu: the same per-(device, stream) workspace
int xform_workspace(cudaStream_t s, int64_t pbytes, int64_t ntick, void** partials, unsigned** tickets) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return XR_ERR_CUDA; }
  std::lock_guard<std::mutex> lock(g_mu);
  Workspace& w = g_ws[{dev, (uintptr_t)s}];
  int st = ensure_ws(w, pbytes, ntick, s);
  if (st) return st;
  *partials = w.partials;
  *tickets = w.tickets;
  return XR_OK;
}
// used by xr_multi.cu: the same per-(device, stream) workspace
int multi_workspace(cudaStream_t s, int64_t pbytes, int64_t ntick, void** partials, unsigned** tickets) {
  return xform_workspace(s, pbytes, ntick, partials, tickets);
}
// used by xr_paper.cu: the partial / RMP buffers of the paper-faithful kernels
int paper_workspace(cudaStream_t s, int64_t bytes, void** buf) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return XR_ERR_CUDA; }
  std::lock_guard<std::mutex> lock(g_mu);
  Workspace& w = g_ws[{dev, (uintptr_t)s}];
  int st = ensure_ws(w, bytes, 0, s);
  if (st) return st;
  *buf = w.partials;
  return XR_OK;
}
// used by xr_heat.cu: the same per-(device, stream) workspace
int heat_workspace(cudaStream_t s, int64_t pbytes, int64_t ntick, void** partials, unsigned** tickets) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return XR_ERR_CUDA; }
  std::lock_guard<std::mutex> lock(g_mu);
  Workspace& w = g_ws[{dev, (uintptr_t)s}];
  int st = ensure_ws(w, pbytes, ntick, s);
  if (st) return st;
  *partials = w.partials;
  *tickets = w.tickets;
  return XR_OK;
}
}  // namespace xr
