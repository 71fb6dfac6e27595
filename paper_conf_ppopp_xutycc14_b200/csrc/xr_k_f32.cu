// xr_k_f32.cu -- explicit instantiation of every legal op for float
// (one translation unit per dtype so the 30 (op, dtype) pairs compile in parallel).
#include "xr_kernels.cuh"

namespace xr {

cudaError_t launch_f32(int op, Plan& p, int num_sms, cudaStream_t s) {
  switch (op) {
    case OP_ADD: return launch_typed<OP_ADD, float>(p, num_sms, s);
    case OP_MUL: return launch_typed<OP_MUL, float>(p, num_sms, s);
    case OP_MAX: return launch_typed<OP_MAX, float>(p, num_sms, s);
    case OP_MIN: return launch_typed<OP_MIN, float>(p, num_sms, s);
    case OP_LAND: return launch_typed<OP_LAND, float>(p, num_sms, s);
    case OP_LOR: return launch_typed<OP_LOR, float>(p, num_sms, s);
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t gather_f32(int op, const void* g, int nranks, int64_t n, void* out, cudaStream_t s) {
  switch (op) {
    case OP_ADD: return launch_gather_typed<OP_ADD, float>(g, nranks, n, out, s);
    case OP_MUL: return launch_gather_typed<OP_MUL, float>(g, nranks, n, out, s);
    case OP_MAX: return launch_gather_typed<OP_MAX, float>(g, nranks, n, out, s);
    case OP_MIN: return launch_gather_typed<OP_MIN, float>(g, nranks, n, out, s);
    case OP_LAND: return launch_gather_typed<OP_LAND, float>(g, nranks, n, out, s);
    case OP_LOR: return launch_gather_typed<OP_LOR, float>(g, nranks, n, out, s);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace xr
