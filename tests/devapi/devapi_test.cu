// tests/devapi/devapi_test.cu -- TEST of the public device API
// (include/xreduce_device.cuh).  Uses ONLY the public header.
//  devapi_gmem: a kernel that reserves ALL its shared memory for its own work
//   (it stages each tile of x through a 200 KiB dynamic buffer, like a blocked
//   matmul would) and therefore reduces with xr::grid_reduce_gmem (no smem).
//  devapi_block: per-block results with xr::block_reduce (segmented output).
#include <cstdint>

#include "../../include/xreduce_device.cuh"

namespace {
constexpr int kThreads = 256;
constexpr int kTileBytes = 200 * 1024;

template <int OP, typename T>
__global__ void __launch_bounds__(kThreads) gmem_kernel(const T* x, int64_t n, T* out,
                                                        xr::GmemWorkspace<typename xr::Op<OP, T>::Acc> ws, int ifo) {
  using O = xr::Op<OP, T>;
  extern __shared__ __align__(16) unsigned char tile[];  // reserved by "the user's computation"
  T* t = reinterpret_cast<T*>(tile);
  constexpr int64_t per = kTileBytes / sizeof(T);
  typename O::Acc v = O::identity();
  for (int64_t base = (int64_t)blockIdx.x * per; base < n; base += (int64_t)gridDim.x * per) {
    const int64_t m = n - base < per ? n - base : per;
    for (int64_t i = threadIdx.x; i < m; i += kThreads) t[i] = x[base + i];
    __syncthreads();
    for (int64_t i = threadIdx.x; i < m; i += kThreads) v = O::combine(v, O::lift(t[i]));
    __syncthreads();
  }
  xr::grid_reduce_gmem<OP, T>(v, ws, out, ifo != 0);
}

template <int OP, typename T>
__global__ void __launch_bounds__(kThreads) block_kernel(const T* x, int64_t seg, T* out) {
  using O = xr::Op<OP, T>;
  __shared__ typename O::Acc slots[32];
  typename O::Acc v = O::identity();
  for (int64_t i = threadIdx.x; i < seg; i += kThreads) v = O::combine(v, O::lift(x[blockIdx.x * seg + i]));
  v = xr::block_reduce<OP, T, kThreads>(v, slots);
  if (threadIdx.x == 0) out[blockIdx.x] = O::finish(v);
}

template <int OP, typename T>
int run_gmem(const void* x, int64_t n, void* out, void* wsp, unsigned* ticket, int grid, int ifo) {
  auto k = gmem_kernel<OP, T>;
  if (cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, kTileBytes) != cudaSuccess) return 3;
  xr::GmemWorkspace<typename xr::Op<OP, T>::Acc> ws{static_cast<typename xr::Op<OP, T>::Acc*>(wsp), ticket};
  k<<<grid, kThreads, kTileBytes>>>(static_cast<const T*>(x), n, static_cast<T*>(out), ws, ifo);
  return cudaDeviceSynchronize() == cudaSuccess ? 0 : 3;
}

template <int OP, typename T>
int run_block(const void* x, int64_t nseg, int64_t seg, void* out) {
  block_kernel<OP, T><<<(unsigned)nseg, kThreads>>>(static_cast<const T*>(x), seg, static_cast<T*>(out));
  return cudaDeviceSynchronize() == cudaSuccess ? 0 : 3;
}
}  // namespace

#define DISPATCH(FN, ...)                                                  \
  switch (dtype * 16 + op) {                                               \
    case 0 * 16 + 0: return FN<xr::OP_ADD, int32_t>(__VA_ARGS__);         \
    case 0 * 16 + 6: return FN<xr::OP_BXOR, int32_t>(__VA_ARGS__);        \
    case 1 * 16 + 2: return FN<xr::OP_MAX, int64_t>(__VA_ARGS__);         \
    case 1 * 16 + 7: return FN<xr::OP_LAND, int64_t>(__VA_ARGS__);        \
    case 2 * 16 + 0: return FN<xr::OP_ADD, float>(__VA_ARGS__);           \
    case 2 * 16 + 3: return FN<xr::OP_MIN, float>(__VA_ARGS__);           \
    case 3 * 16 + 0: return FN<xr::OP_ADD, double>(__VA_ARGS__);          \
    case 3 * 16 + 1: return FN<xr::OP_MUL, double>(__VA_ARGS__);          \
    default: return 2;                                                     \
  }

extern "C" int devapi_gmem(int op, int dtype, const void* x, int64_t n, void* out, void* ws, unsigned* ticket,
                           int grid, int ifo) {
  DISPATCH(run_gmem, x, n, out, ws, ticket, grid, ifo)
}
extern "C" int devapi_block(int op, int dtype, const void* x, int64_t nseg, int64_t seg, void* out) {
  DISPATCH(run_block, x, nseg, seg, out)
}
