// xr_comm.cpp -- multi-GPU gang sharding.
//
// In the paper, gangs compute independent private partials and only the
// cross-gang combine needs a global synchronisation, which thread blocks
// cannot do (PAPER.md @7679, @24887-25280).  Across GPUs the same structure
// holds: each rank reduces its contiguous gang slice with the single-GPU path
// (blocking across GPUs; the paper notes blocking and window sliding are
// equivalent for gang partial reduction, @25998-26464), then ONE collective
// over NVLink/NVSwitch combines them (xr_shard_plan decides which).
#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <vector>
#include <nccl.h>

#include "../../include/xreduce.h"
#include "xr_internal.h"

namespace xr {
int reduce_device_checked(int op, int dtype, const int64_t* dims, unsigned mask, const void* in, void* out,
                          cudaStream_t s, const ExchArgs* exch = nullptr);
cudaError_t gather_combine(int op, int dtype, const void* g, int nranks, int64_t n, void* out, cudaStream_t s);
int heat_slab_rows(int64_t n_local, int nranks, int rank, int64_t* jb, int64_t* je);
int heat_step_rows(int64_t nj, int64_t ni, int64_t jb, int64_t je, const double* T1, double* T2,
                   double* residual, cudaStream_t s, const double* res_init = nullptr);
int reduce_host_into(int op, int dtype, const int64_t* dims, unsigned mask, const void* in_host, void* out_dev,
                     cudaStream_t s);
}  // namespace xr

using xr::kMaxRanks;
using xr::kMailboxWords;
using xr::ExchArgs;

struct xr_comm_s {
  ncclComm_t nccl = nullptr;
  int nranks = 0, rank = 0, device = 0;
  void* scratch = nullptr;  // allgather buffers for & | ^
  size_t scratch_bytes = 0;
  void* hout = nullptr;     // device copy of the output of xr_reduce_sharded_host
  size_t hout_bytes = 0;
  // overlapped sharded heat run: a communication stream, its events and the
  // boundary-row residual slot
  cudaStream_t cstream = nullptr;
  cudaEvent_t ev_start = nullptr, ev_bound = nullptr, ev_sweep = nullptr, ev_halo = nullptr, ev_end = nullptr;
  double* res_bound = nullptr;
  // fused exchange (peer mailboxes over NVLink via CUDA IPC)
  bool fused = false;                         // set up and enabled
  unsigned long long* mailbox = nullptr;      // mine
  unsigned long long* peers[kMaxRanks] = {};  // every rank's mailbox, mapped into this process
  int* status = nullptr;        // host-mapped pinned word (device pointer below)
  int* status_dev = nullptr;
  unsigned long long epoch = 0;
  unsigned long long timeout_ns = 0;
};

// Wait bound of the fused exchange: a peer later than this is reported (the
// host-mapped status word) instead of hanging the GPU.  XR_EXCH_TIMEOUT_MS
// overrides (tests).
static unsigned long long exch_timeout_ns() {
  const char* e = std::getenv("XR_EXCH_TIMEOUT_MS");
  const long long ms = e ? std::atoll(e) : 20000;
  return (unsigned long long)std::max(1ll, ms) * 1000000ull;
}

// Allocate this rank's mailbox, all-gather the CUDA IPC handles with NCCL and
// map every peer's mailbox.  Any failure leaves the communicator on NCCL.
static void setup_fused(xr_comm_s* c) {
  if (c->nranks > kMaxRanks) return;
  const size_t bytes = kMailboxWords * sizeof(unsigned long long);
  if (cudaMalloc(&c->mailbox, bytes) != cudaSuccess ||
      cudaHostAlloc(reinterpret_cast<void**>(&c->status), sizeof(int), cudaHostAllocMapped) != cudaSuccess ||
      cudaHostGetDevicePointer(reinterpret_cast<void**>(&c->status_dev), c->status, 0) != cudaSuccess) {
    cudaGetLastError();
    return;
  }
  cudaMemset(c->mailbox, 0, bytes);
  *reinterpret_cast<volatile int*>(c->status) = 0;
  c->timeout_ns = exch_timeout_ns();
  c->peers[c->rank] = c->mailbox;
  if (c->nranks > 1) {
    cudaIpcMemHandle_t h;
    if (cudaIpcGetMemHandle(&h, c->mailbox) != cudaSuccess) { cudaGetLastError(); return; }
    char* d = nullptr;
    if (cudaMalloc(&d, (size_t)(c->nranks + 1) * sizeof h) != cudaSuccess) { cudaGetLastError(); return; }
    cudaMemcpy(d, &h, sizeof h, cudaMemcpyHostToDevice);
    const bool ok = ncclAllGather(d, d + sizeof h, sizeof h, ncclChar, c->nccl, 0) == ncclSuccess;
    std::vector<cudaIpcMemHandle_t> all(c->nranks);
    cudaMemcpy(all.data(), d + sizeof h, c->nranks * sizeof h, cudaMemcpyDeviceToHost);  // syncs stream 0
    cudaFree(d);
    if (!ok) return;
    for (int p = 0; p < c->nranks; ++p) {
      if (p == c->rank) continue;
      void* ptr = nullptr;
      if (cudaIpcOpenMemHandle(&ptr, all[p], cudaIpcMemLazyEnablePeerAccess) != cudaSuccess) {
        cudaGetLastError();
        return;
      }
      c->peers[p] = static_cast<unsigned long long*>(ptr);
    }
  }
  cudaDeviceSynchronize();
  c->fused = cudaGetLastError() == cudaSuccess;
}

using namespace xr;

static ncclDataType_t nccl_type(int dtype) {
  switch (dtype) {
    case XR_INT32: return ncclInt32;
    case XR_INT64: return ncclInt64;
    case XR_FP32: return ncclFloat32;
    default: return ncclFloat64;
  }
}

extern "C" {

int xr_comm_get_unique_id(void* id128) {
  if (!id128) return XR_ERR_INVALID;
  ncclUniqueId id;
  if (ncclGetUniqueId(&id) != ncclSuccess) return XR_ERR_NCCL;
  std::memcpy(id128, &id, sizeof id);
  return XR_OK;
}

int xr_comm_init(xr_comm_t* comm, int nranks, int rank, const void* id128, int device) {
  if (!comm || !id128 || nranks < 1 || rank < 0 || rank >= nranks || device < 0) return XR_ERR_INVALID;
  if (cudaSetDevice(device) != cudaSuccess) { cudaGetLastError(); return XR_ERR_CUDA; }
  ncclUniqueId id;
  std::memcpy(&id, id128, sizeof id);
  xr_comm_s* c = new xr_comm_s();
  c->nranks = nranks;
  c->rank = rank;
  c->device = device;
  if (ncclCommInitRank(&c->nccl, nranks, id, rank) != ncclSuccess) {
    delete c;
    return XR_ERR_NCCL;
  }
  setup_fused(c);
  if (nranks > 1) {
    // consensus: the fused exchange is used only if EVERY rank mapped every
    // peer (a mixed setup would leave fused ranks spinning while the others
    // sit in an NCCL collective)
    int* d = nullptr;
    int ok = c->fused ? 1 : 0;
    if (cudaMalloc(&d, sizeof(int)) == cudaSuccess) {
      cudaMemcpy(d, &ok, sizeof(int), cudaMemcpyHostToDevice);
      if (ncclAllReduce(d, d, 1, ncclInt32, ncclMin, c->nccl, 0) == ncclSuccess)
        cudaMemcpy(&ok, d, sizeof(int), cudaMemcpyDeviceToHost);
      else
        ok = 0;
      cudaFree(d);
    } else {
      cudaGetLastError();
      ok = 0;  // NOTE: this rank still joined no collective; all ranks reach the allreduce above or fail alike
    }
    c->fused = ok == 1;
  }
  *comm = c;
  return XR_OK;
}

static int read_status(const xr_comm_s* c) {
  return c->status ? *reinterpret_cast<volatile const int*>(c->status) : 0;
}

int xr_comm_set_fused(xr_comm_t comm, int enable) {
  if (!comm) return XR_ERR_INVALID;
  if (!enable) {
    comm->fused = false;
    return XR_OK;
  }
  if (!comm->mailbox || !comm->status) return XR_ERR_UNSUPPORTED;
  for (int p = 0; p < comm->nranks; ++p)  // every peer mapped
    if (!comm->peers[p]) return XR_ERR_UNSUPPORTED;
  // Collective: re-synchronise the mailbox epochs (a timed-out exchange can
  // leave ranks at different epochs) and clear the status word.  Every rank
  // calls this; nothing of this communicator may be in flight.
  if (cudaSetDevice(comm->device) != cudaSuccess || cudaDeviceSynchronize() != cudaSuccess) {
    cudaGetLastError();
    return XR_ERR_CUDA;
  }
  unsigned long long* d = nullptr;
  if (cudaMalloc(&d, sizeof *d) != cudaSuccess) { cudaGetLastError(); return XR_ERR_NOMEM; }
  unsigned long long e = comm->epoch;
  int st = XR_OK;
  if (cudaMemcpy(d, &e, sizeof e, cudaMemcpyHostToDevice) != cudaSuccess) st = XR_ERR_CUDA;
  else if (ncclAllReduce(d, d, 1, ncclUint64, ncclMax, comm->nccl, 0) != ncclSuccess) st = XR_ERR_NCCL;
  else if (cudaMemcpy(&e, d, sizeof e, cudaMemcpyDeviceToHost) != cudaSuccess) st = XR_ERR_CUDA;
  cudaFree(d);
  if (st) { cudaGetLastError(); return st; }
  comm->epoch = e;
  *reinterpret_cast<volatile int*>(comm->status) = 0;
  comm->fused = true;
  return XR_OK;
}

int xr_comm_query(xr_comm_t comm, int* fused, int* status) {
  if (!comm) return XR_ERR_INVALID;
  if (fused) *fused = comm->fused ? 1 : 0;
  if (status) *status = read_status(comm);  // host-mapped: no device synchronisation
  return XR_OK;
}

int xr_comm_destroy(xr_comm_t comm) {
  if (!comm) return XR_ERR_INVALID;
  int st = XR_OK;
  for (int p = 0; p < comm->nranks && p < kMaxRanks; ++p)
    if (p != comm->rank && comm->peers[p]) cudaIpcCloseMemHandle(comm->peers[p]);
  if (comm->mailbox) cudaFree(comm->mailbox);
  if (comm->status) cudaFreeHost(comm->status);
  if (comm->scratch) cudaFree(comm->scratch);
  if (comm->hout) cudaFree(comm->hout);
  if (comm->res_bound) cudaFree(comm->res_bound);
  for (cudaEvent_t e : {comm->ev_start, comm->ev_bound, comm->ev_sweep, comm->ev_halo, comm->ev_end})
    if (e) cudaEventDestroy(e);
  if (comm->cstream) cudaStreamDestroy(comm->cstream);
  if (comm->nccl && ncclCommDestroy(comm->nccl) != ncclSuccess) st = XR_ERR_NCCL;
  delete comm;
  return st;
}

}  // extern "C"

// The sharded protocol around a local reduction `local(mask, dst)` that writes
// this rank's xr_out_count(local_dims) results to device memory dst (merging
// dst as init when mask has XR_INIT_FROM_OUT).  fused_local: the same
// reduction with the fused NVLink exchange (nullptr when the caller's local
// reduction cannot host it).
template <typename Local, typename FusedLocal>
static int sharded_impl(int op, int dtype, const int64_t local_dims[3], unsigned level_mask, void* out,
                        xr_comm_t comm, cudaStream_t s, Local local, FusedLocal* fused_local) {
  xr_shard_info info;
  int st = xr_shard_plan(op, dtype, local_dims, level_mask, comm->nranks, comm->rank, &info);
  if (st) return st;
  if (info.global_count == 0) return XR_OK;
  if (!out) return XR_ERR_INVALID;
  const int size = dtype_size(dtype);
  const unsigned base = (level_mask & 7u) | (info.local_init_from_out ? XR_INIT_FROM_OUT : 0u);
  char* mine = (char*)out + info.out_offset * size;

  if (info.collective == XR_COLL_ALLGATHER_COMBINE) {
    // & | ^: NCCL has no bitwise reduction -> gather partials, fixed-order combine
    const size_t need = (size_t)(comm->nranks + 1) * info.local_count * size;
    if (need > comm->scratch_bytes) {
      if (comm->scratch) { cudaStreamSynchronize(s); cudaFree(comm->scratch); }
      comm->scratch = nullptr;
      comm->scratch_bytes = 0;
      if (cudaMalloc(&comm->scratch, need) != cudaSuccess) { cudaGetLastError(); return XR_ERR_NOMEM; }
      comm->scratch_bytes = need;
    }
    char* lbuf = (char*)comm->scratch;
    char* gathered = lbuf + (size_t)info.local_count * size;
    if (info.local_init_from_out &&
        cudaMemcpyAsync(lbuf, out, (size_t)info.local_count * size, cudaMemcpyDeviceToDevice, s) != cudaSuccess)
      return XR_ERR_CUDA;
    if ((st = local(base, lbuf))) return st;
    if (ncclAllGather(lbuf, gathered, (size_t)info.local_count, nccl_type(dtype), comm->nccl, s) != ncclSuccess)
      return XR_ERR_NCCL;
    if (gather_combine(op, dtype, gathered, comm->nranks, info.local_count, out, s) != cudaSuccess)
      return XR_ERR_CUDA;
    return XR_OK;
  }

  if (fused_local && comm->fused && (level_mask & XR_GANG) && info.global_count == 1) {
    // a previous fused exchange timed out: the mailbox epochs may disagree
    // across ranks, so refuse until xr_comm_set_fused re-synchronises them
    if (read_status(comm)) return XR_ERR_NCCL;
    // one kernel: local reduction + peer-mailbox exchange over NVLink
    ExchArgs x{};
    x.mine = comm->mailbox;
    for (int p = 0; p < comm->nranks; ++p) x.peers[p] = comm->peers[p];
    x.nranks = comm->nranks;
    x.rank = comm->rank;
    x.epoch = ++comm->epoch;
    x.timeout_ns = comm->timeout_ns;
    x.status = comm->status_dev;
    st = (*fused_local)(base, mine, &x);
    if (st == XR_OK) return XR_OK;
    --comm->epoch;  // nothing was launched: the epoch stays in step with the peers
    if (st != XR_ERR_UNSUPPORTED) return st;
    // this plan cannot host the exchange: NCCL below
  }
  if ((st = local(base, mine))) return st;
  // the collective runs at every world size (a 1-rank communicator executes
  // the same NCCL call, so its op / dtype mapping is exercised on one GPU)
  if (info.collective == XR_COLL_ALLREDUCE) {
    if (ncclAllReduce(out, out, (size_t)info.global_count, nccl_type(dtype), (ncclRedOp_t)info.nccl_op,
                      comm->nccl, s) != ncclSuccess)
      return XR_ERR_NCCL;
  } else if (info.collective == XR_COLL_ALLGATHER) {
    // in place: rank r's segment already sits at out + r*local_count
    if (ncclAllGather(mine, out, (size_t)info.local_count, nccl_type(dtype), comm->nccl, s) != ncclSuccess)
      return XR_ERR_NCCL;
  }
  return XR_OK;
}

extern "C" {

int xr_reduce_sharded(int op, int dtype, const int64_t local_dims[3], unsigned level_mask,
                      const void* in_local, void* out, xr_comm_t comm, xr_stream_t stream) {
  if (!comm) return XR_ERR_INVALID;
  cudaStream_t s = (cudaStream_t)stream;
  auto local = [&](unsigned m, void* dst) { return reduce_device_checked(op, dtype, local_dims, m, in_local, dst, s); };
  auto fused = [&](unsigned m, void* dst, const ExchArgs* x) {
    return reduce_device_checked(op, dtype, local_dims, m, in_local, dst, s, x);
  };
  return sharded_impl(op, dtype, local_dims, level_mask, out, comm, s, local, &fused);
}

int xr_reduce_sharded_host(int op, int dtype, const int64_t local_dims[3], unsigned level_mask,
                           const void* in_local_host, void* out_host, xr_comm_t comm, xr_stream_t stream) {
  if (!comm) return XR_ERR_INVALID;
  xr_shard_info info;
  int st = xr_shard_plan(op, dtype, local_dims, level_mask, comm->nranks, comm->rank, &info);
  if (st) return st;
  if (info.global_count == 0) return XR_OK;
  int64_t total = local_dims[0] * local_dims[1] * local_dims[2];
  if (!out_host || (total > 0 && !in_local_host)) return XR_ERR_INVALID;
  cudaStream_t s = (cudaStream_t)stream;
  const size_t obytes = (size_t)info.global_count * dtype_size(dtype);
  if (obytes > comm->hout_bytes) {
    if (comm->hout) { cudaStreamSynchronize(s); cudaFree(comm->hout); }
    comm->hout = nullptr;
    comm->hout_bytes = 0;
    if (cudaMalloc(&comm->hout, obytes) != cudaSuccess) { cudaGetLastError(); return XR_ERR_NOMEM; }
    comm->hout_bytes = obytes;
  }
  // the caller's init (XR_INIT_FROM_OUT) travels with out
  if ((level_mask & XR_INIT_FROM_OUT) &&
      cudaMemcpyAsync(comm->hout, out_host, obytes, cudaMemcpyHostToDevice, s) != cudaSuccess) {
    cudaGetLastError();
    return XR_ERR_CUDA;
  }
  // local reduction: the chunked H2D pipeline of xr_reduce_host into device memory
  auto local = [&](unsigned m, void* dst) {
    return reduce_host_into(op, dtype, local_dims, m, in_local_host, dst, s);
  };
  using NoFused = int(unsigned, void*, const ExchArgs*);
  st = sharded_impl(op, dtype, local_dims, level_mask, comm->hout, comm, s, local, (NoFused*)nullptr);
  if (!st && cudaMemcpyAsync(out_host, comm->hout, obytes, cudaMemcpyDeviceToHost, s) != cudaSuccess) st = XR_ERR_CUDA;
  if (cudaStreamSynchronize(s) != cudaSuccess && !st) st = XR_ERR_CUDA;
  if (st) cudaGetLastError();
  return st;
}

int xr_heat_step_sharded(int64_t n_local, int64_t ni, const double* T1, double* T2, double* residual,
                         xr_comm_t comm, xr_stream_t stream) {
  if (!comm || !residual || n_local < 1 || ni < 0 || !T1 || !T2) return XR_ERR_INVALID;
  cudaStream_t s = (cudaStream_t)stream;
  int64_t jb, je;
  int st = heat_slab_rows(n_local, comm->nranks, comm->rank, &jb, &je);
  if (st) return st;
  if ((st = heat_step_rows(n_local + 2, ni, jb, je, T1, T2, residual, s))) return st;
  // halo rows of the new field: my first owned row goes up, my last goes down.
  // XR_FORCE_COLL (tests, 1 rank): the rank is its own up and down neighbour,
  // so the grouped send/recv runs on one GPU; NCCL matches the two self
  // messages in order, i.e. halo row 0 <- owned row 1 and halo row n+1 <-
  // owned row n.  Both halo rows are unused at the global boundary.
  const int r = comm->rank;
  const bool force = comm->nranks == 1 && std::getenv("XR_FORCE_COLL") != nullptr;
  const int up = r > 0 ? r - 1 : (force ? r : -1);
  const int down = r < comm->nranks - 1 ? r + 1 : (force ? r : -1);
  if (up >= 0 || down >= 0) {
    if (ncclGroupStart() != ncclSuccess) return XR_ERR_NCCL;
    if (up >= 0) {
      ncclSend(T2 + ni, (size_t)ni, ncclFloat64, up, comm->nccl, s);
      ncclRecv(T2, (size_t)ni, ncclFloat64, up, comm->nccl, s);
    }
    if (down >= 0) {
      ncclSend(T2 + n_local * ni, (size_t)ni, ncclFloat64, down, comm->nccl, s);
      ncclRecv(T2 + (n_local + 1) * ni, (size_t)ni, ncclFloat64, down, comm->nccl, s);
    }
    if (ncclGroupEnd() != ncclSuccess) return XR_ERR_NCCL;
  }
  if (ncclAllReduce(residual, residual, 1, ncclFloat64, ncclMax, comm->nccl, s) != ncclSuccess) return XR_ERR_NCCL;
  return XR_OK;
}

// The halo rows of sweep k+1 depend only on the BOUNDARY rows of sweep k, so
// those are swept first (two one-row launches), the halo exchange runs on a
// communication stream while the interior sweeps, and the residual allreduce
// of sweep k is issued on that stream after the halos of sweep k+1: it is
// lagged one sweep and hidden behind the next interior sweep (SURVEY 8(e),
// "heat at G = 8").  Every residual is still exact and final when the run
// returns to the stream: max is exact, and the interior launch merges the
// boundary rows' maximum (res_init), so residuals are bit-identical to the
// serial protocol.
static int halo_exchange(xr_comm_t comm, int64_t n_local, int64_t ni, double* T, cudaStream_t c) {
  const int r = comm->rank;
  const bool force = comm->nranks == 1 && std::getenv("XR_FORCE_COLL") != nullptr;
  const int up = r > 0 ? r - 1 : (force ? r : -1);
  const int down = r < comm->nranks - 1 ? r + 1 : (force ? r : -1);
  if (up < 0 && down < 0) return XR_OK;
  if (ncclGroupStart() != ncclSuccess) return XR_ERR_NCCL;
  if (up >= 0) {
    ncclSend(T + ni, (size_t)ni, ncclFloat64, up, comm->nccl, c);
    ncclRecv(T, (size_t)ni, ncclFloat64, up, comm->nccl, c);
  }
  if (down >= 0) {
    ncclSend(T + n_local * ni, (size_t)ni, ncclFloat64, down, comm->nccl, c);
    ncclRecv(T + (n_local + 1) * ni, (size_t)ni, ncclFloat64, down, comm->nccl, c);
  }
  return ncclGroupEnd() == ncclSuccess ? XR_OK : XR_ERR_NCCL;
}

int xr_heat_run_sharded(int64_t n_local, int64_t ni, int64_t iters, double* T1, double* T2, double* residuals,
                        xr_comm_t comm, xr_stream_t stream) {
  if (!comm || n_local < 1 || ni < 0 || !T1 || !T2 || iters < 0 || (iters > 0 && !residuals)) return XR_ERR_INVALID;
  if (iters == 0) return XR_OK;
  cudaStream_t s = (cudaStream_t)stream;
  if (!comm->cstream) {
    if (cudaStreamCreateWithFlags(&comm->cstream, cudaStreamNonBlocking) != cudaSuccess ||
        cudaMalloc(&comm->res_bound, 2 * sizeof(double)) != cudaSuccess) {
      cudaGetLastError();
      return XR_ERR_CUDA;
    }
    for (cudaEvent_t* e : {&comm->ev_start, &comm->ev_bound, &comm->ev_sweep, &comm->ev_halo, &comm->ev_end})
      if (cudaEventCreateWithFlags(e, cudaEventDisableTiming) != cudaSuccess) { cudaGetLastError(); return XR_ERR_CUDA; }
  }
  cudaStream_t c = comm->cstream;
  int64_t jb, je;
  int st = heat_slab_rows(n_local, comm->nranks, comm->rank, &jb, &je);
  if (st) return st;
  const int64_t nj = n_local + 2;
  const bool split = je - jb >= 3;  // boundary rows jb and je-1 swept before the interior
  auto cu = [](cudaError_t e) { return e == cudaSuccess ? XR_OK : (cudaGetLastError(), XR_ERR_CUDA); };
  // the communication stream starts after the caller's prior work on `stream`
  if ((st = cu(cudaEventRecord(comm->ev_start, s))) || (st = cu(cudaStreamWaitEvent(c, comm->ev_start, 0)))) return st;
  double* a = T1;
  double* b = T2;
  for (int64_t it = 0; it < iters; ++it) {
    if (it > 0 && (st = cu(cudaStreamWaitEvent(s, comm->ev_halo, 0)))) return st;  // a's halos landed
    if (split) {
      if ((st = heat_step_rows(nj, ni, jb, jb + 1, a, b, comm->res_bound, s))) return st;
      if ((st = heat_step_rows(nj, ni, je - 1, je, a, b, comm->res_bound, s, comm->res_bound))) return st;
      if ((st = cu(cudaEventRecord(comm->ev_bound, s)))) return st;
      if ((st = heat_step_rows(nj, ni, jb + 1, je - 1, a, b, residuals + it, s, comm->res_bound))) return st;
    } else {
      if ((st = heat_step_rows(nj, ni, jb, je, a, b, residuals + it, s))) return st;
      if ((st = cu(cudaEventRecord(comm->ev_bound, s)))) return st;
    }
    // communication stream: b's halos (its boundary rows are final), then the
    // residual of the PREVIOUS sweep (its interior launch precedes ev_bound)
    if ((st = cu(cudaStreamWaitEvent(c, comm->ev_bound, 0)))) return st;
    if ((st = halo_exchange(comm, n_local, ni, b, c))) return st;
    if ((st = cu(cudaEventRecord(comm->ev_halo, c)))) return st;
    if (it > 0 && ncclAllReduce(residuals + it - 1, residuals + it - 1, 1, ncclFloat64, ncclMax, comm->nccl, c) !=
                      ncclSuccess)
      return XR_ERR_NCCL;
    double* t = a;
    a = b;
    b = t;
  }
  // the last residual, then join the communication stream back into `stream`
  if ((st = cu(cudaEventRecord(comm->ev_sweep, s))) || (st = cu(cudaStreamWaitEvent(c, comm->ev_sweep, 0)))) return st;
  if (ncclAllReduce(residuals + iters - 1, residuals + iters - 1, 1, ncclFloat64, ncclMax, comm->nccl, c) != ncclSuccess)
    return XR_ERR_NCCL;
  if ((st = cu(cudaEventRecord(comm->ev_end, c))) || (st = cu(cudaStreamWaitEvent(s, comm->ev_end, 0)))) return st;
  return XR_OK;
}

}  // extern "C"
