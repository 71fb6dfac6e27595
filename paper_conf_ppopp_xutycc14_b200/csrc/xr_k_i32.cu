// xr_k_i32.cu -- explicit instantiation of every legal op for int32_t
// (one translation unit per dtype so the 30 (op, dtype) pairs compile in parallel).
#include "xr_kernels.cuh"

namespace xr {

cudaError_t launch_i32(int op, Plan& p, int num_sms, cudaStream_t s) {
  switch (op) {
    case OP_ADD: return launch_typed<OP_ADD, int32_t>(p, num_sms, s);
    case OP_MUL: return launch_typed<OP_MUL, int32_t>(p, num_sms, s);
    case OP_MAX: return launch_typed<OP_MAX, int32_t>(p, num_sms, s);
    case OP_MIN: return launch_typed<OP_MIN, int32_t>(p, num_sms, s);
    case OP_BAND: return launch_typed<OP_BAND, int32_t>(p, num_sms, s);
    case OP_BOR: return launch_typed<OP_BOR, int32_t>(p, num_sms, s);
    case OP_BXOR: return launch_typed<OP_BXOR, int32_t>(p, num_sms, s);
    case OP_LAND: return launch_typed<OP_LAND, int32_t>(p, num_sms, s);
    case OP_LOR: return launch_typed<OP_LOR, int32_t>(p, num_sms, s);
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t gather_i32(int op, const void* g, int nranks, int64_t n, void* out, cudaStream_t s) {
  switch (op) {
    case OP_ADD: return launch_gather_typed<OP_ADD, int32_t>(g, nranks, n, out, s);
    case OP_MUL: return launch_gather_typed<OP_MUL, int32_t>(g, nranks, n, out, s);
    case OP_MAX: return launch_gather_typed<OP_MAX, int32_t>(g, nranks, n, out, s);
    case OP_MIN: return launch_gather_typed<OP_MIN, int32_t>(g, nranks, n, out, s);
    case OP_BAND: return launch_gather_typed<OP_BAND, int32_t>(g, nranks, n, out, s);
    case OP_BOR: return launch_gather_typed<OP_BOR, int32_t>(g, nranks, n, out, s);
    case OP_BXOR: return launch_gather_typed<OP_BXOR, int32_t>(g, nranks, n, out, s);
    case OP_LAND: return launch_gather_typed<OP_LAND, int32_t>(g, nranks, n, out, s);
    case OP_LOR: return launch_gather_typed<OP_LOR, int32_t>(g, nranks, n, out, s);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace xr
