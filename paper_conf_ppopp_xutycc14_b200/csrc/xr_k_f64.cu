// xr_k_f64.cu -- explicit instantiation of every legal op for double
// (one translation unit per dtype so the 30 (op, dtype) pairs compile in parallel).
#include "xr_kernels.cuh"

namespace xr {

cudaError_t launch_f64(int op, Plan& p, int num_sms, cudaStream_t s) {
  switch (op) {
    case OP_ADD: return launch_typed<OP_ADD, double>(p, num_sms, s);
    case OP_MUL: return launch_typed<OP_MUL, double>(p, num_sms, s);
    case OP_MAX: return launch_typed<OP_MAX, double>(p, num_sms, s);
    case OP_MIN: return launch_typed<OP_MIN, double>(p, num_sms, s);
    case OP_LAND: return launch_typed<OP_LAND, double>(p, num_sms, s);
    case OP_LOR: return launch_typed<OP_LOR, double>(p, num_sms, s);
    default: return cudaErrorInvalidValue;
  }
}

cudaError_t gather_f64(int op, const void* g, int nranks, int64_t n, void* out, cudaStream_t s) {
  switch (op) {
    case OP_ADD: return launch_gather_typed<OP_ADD, double>(g, nranks, n, out, s);
    case OP_MUL: return launch_gather_typed<OP_MUL, double>(g, nranks, n, out, s);
    case OP_MAX: return launch_gather_typed<OP_MAX, double>(g, nranks, n, out, s);
    case OP_MIN: return launch_gather_typed<OP_MIN, double>(g, nranks, n, out, s);
    case OP_LAND: return launch_gather_typed<OP_LAND, double>(g, nranks, n, out, s);
    case OP_LOR: return launch_gather_typed<OP_LOR, double>(g, nranks, n, out, s);
    default: return cudaErrorInvalidValue;
  }
}

}  // namespace xr
