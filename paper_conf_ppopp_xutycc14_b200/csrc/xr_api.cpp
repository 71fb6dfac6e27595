// xr_api.cpp -- the C ABI (include/xreduce.h): validation, workspace, dispatch.
// Validation never touches CUDA, so every status path is testable on a CPU
// machine (tests/test_abi.py).
#include <atomic>
#include <cstring>
#include <map>
#include <mutex>
#include <utility>
#include <vector>

#include "../../include/xreduce.h"
#include "xr_internal.h"

namespace xr {

static std::atomic<int64_t> g_launches{0};
void count_launch() { g_launches.fetch_add(1, std::memory_order_relaxed); }

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
  p.col.in = in; p.col.out = out; p.col.partials = w.partials; p.col.tickets = w.tickets;
  p.col.init_from_out = ifo;
  p.elt.in = in; p.elt.out = out; p.elt.init_from_out = ifo;
  p.rkr.in = in; p.rkr.out = out; p.rkr.partials = w.partials; p.rkr.tickets = w.tickets;
  p.rkr.sched = sched; p.rkr.init_from_out = ifo;
  if (p.kernel == K_COLTMA && !make_col_tmap(&p.tmap, dtype, in, p.col.B, p.col.R, p.col.K)) {
    // no tensor-map support: re-plan without TMA (same workspace bound or smaller)
    return XR_ERR_CUDA;
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
struct Staging {
  void* in = nullptr;
  size_t in_bytes = 0;
  void* out = nullptr;
  size_t out_bytes = 0;
};
static std::map<int, Staging> g_stage;

static int grow(void** p, size_t* have, size_t need) {
  if (need <= *have) return XR_OK;
  if (*p) { cudaDeviceSynchronize(); cudaFree(*p); }
  *p = nullptr;
  *have = 0;
  if (cudaMalloc(p, need) != cudaSuccess) { cudaGetLastError(); return XR_ERR_NOMEM; }
  *have = need;
  return XR_OK;
}

}  // namespace xr

using namespace xr;

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
  if (p.kernel == K_STREAM || p.kernel == K_COLTMA || p.kernel == K_ROWS || p.kernel == K_RKR) ctas = std::min<int64_t>(p.units, (int64_t)num_sms * 3);
  if (p.kernel == K_SEG && p.group < p.block) ctas = (p.units + p.block / p.group - 1) / (p.block / p.group);
  if (p.kernel == K_FILL || p.kernel == K_IDENT) ctas = (p.units + kBlock - 1) / kBlock;
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
    if (kv.second.in) cudaFree(kv.second.in);
    if (kv.second.out) cudaFree(kv.second.out);
  }
  g_stage.clear();
  cudaGetLastError();
  return XR_OK;
}

int64_t xr_launch_count(void) { return g_launches.load(); }

int xr_reduce_host(int op, int dtype, const int64_t nest_dims[3], unsigned level_mask,
                   const void* in_host, void* out_host, xr_stream_t stream) {
  int64_t total = 0, count = 0;
  int st = validate(op, dtype, nest_dims, level_mask, &total, &count);
  if (st) return st;
  if (count == 0) return XR_OK;
  if (!out_host || (total > 0 && !in_host)) return XR_ERR_INVALID;
  const int size = dtype_size(dtype);
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return XR_ERR_CUDA; }
  void* din;
  void* dout;
  {
    std::lock_guard<std::mutex> lock(g_mu);
    Staging& sg = g_stage[dev];
    if ((st = grow(&sg.in, &sg.in_bytes, (size_t)std::max<int64_t>(total * size, 16)))) return st;
    if ((st = grow(&sg.out, &sg.out_bytes, (size_t)count * size))) return st;
    din = sg.in;
    dout = sg.out;
  }
  cudaStream_t s = (cudaStream_t)stream;
  if ((level_mask & XR_INIT_FROM_OUT) &&
      cudaMemcpyAsync(dout, out_host, (size_t)count * size, cudaMemcpyHostToDevice, s) != cudaSuccess)
    return XR_ERR_CUDA;
  if (total > 0 && cudaMemcpyAsync(din, in_host, (size_t)total * size, cudaMemcpyHostToDevice, s) != cudaSuccess)
    return XR_ERR_CUDA;
  st = reduce_device(op, dtype, nest_dims, level_mask, din, dout, s);
  if (st) return st;
  if (cudaMemcpyAsync(out_host, dout, (size_t)count * size, cudaMemcpyDeviceToHost, s) != cudaSuccess)
    return XR_ERR_CUDA;
  if (cudaStreamSynchronize(s) != cudaSuccess) return XR_ERR_CUDA;
  return XR_OK;
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
  // each spins on its mailbox until all the others published (real protocol)
  for (int r = 0; r < nranks && !st; ++r) {
    ExchArgs x{};
    x.mine = mb + (size_t)r * kMailboxWords;
    for (int p = 0; p < nranks; ++p) x.peers[p] = mb + (size_t)p * kMailboxWords;
    x.nranks = nranks;
    x.rank = r;
    x.epoch = 1;
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
