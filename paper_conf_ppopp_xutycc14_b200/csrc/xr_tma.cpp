// xr_tma.cpp -- host side of the TMA column path: encode the 3-D tensor map
// (K, R, B) with the driver's cuTensorMapEncodeTiled, fetched once through
// cudaGetDriverEntryPoint (no link-time dependency on libcuda).
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdlib>
#include <mutex>

#include "../../include/xreduce.h"
#include "xr_internal.h"

namespace xr {

static PFN_cuTensorMapEncodeTiled_v12000 encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  static std::once_flag once;
  std::call_once(once, [] {
    void* p = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(p);
    else
      cudaGetLastError();
  });
  return fn;
}

bool make_col_tmap(CUtensorMap* m, int dtype, const void* in, int64_t B, int64_t R, int64_t K, int box_bytes) {
  if (std::getenv("XR_TEST_TMAP_FAIL") != nullptr) return false;  // test hook: the re-plan fallback
  auto fn = encode_fn();
  if (!fn) return false;
  const int size = dtype_size(dtype);
  CUtensorMapDataType t;
  switch (dtype) {
    case XR_INT32: t = CU_TENSOR_MAP_DATA_TYPE_INT32; break;
    case XR_INT64: t = CU_TENSOR_MAP_DATA_TYPE_INT64; break;
    case XR_FP32: t = CU_TENSOR_MAP_DATA_TYPE_FLOAT32; break;
    default: t = CU_TENSOR_MAP_DATA_TYPE_FLOAT64; break;
  }
  const cuuint64_t dims[3] = {(cuuint64_t)K, (cuuint64_t)R, (cuuint64_t)B};
  const cuuint64_t strides[2] = {(cuuint64_t)(K * size), (cuuint64_t)(R * K * size)};
  const cuuint32_t box[3] = {(cuuint32_t)(box_bytes / size), (cuuint32_t)(kStageBytes / box_bytes), 1u};
  const cuuint32_t estr[3] = {1u, 1u, 1u};
  CUresult r = fn(m, t, 3, const_cast<void*>(in), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                  CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  return r == CUDA_SUCCESS;
}

}  // namespace xr
