// DEVICE-class plans (row a9, north star): pack -> all-to-all over NVLink -> unpack.
#include <cuda_runtime.h>

#include "ll_internal.hpp"

namespace ll {

void plan_device(ConvPlan& P, const ll_plan_opts* opts) {
  if (!opts || !opts->comm) fail(LL_ERR_INVALID_ARG, "DEVICE plans require opts->comm (P mixes device bits)");
  fail(LL_ERR_UNSUPPORTED, "DEVICE plans: not built yet");
}

ll_status device_convert(const ConvPlan& P, const void* src, void* dst, void* ws, cudaStream_t st) {
  (void)P; (void)src; (void)dst; (void)ws; (void)st;
  fail(LL_ERR_UNSUPPORTED, "DEVICE plans: not built yet");
}

}  // namespace ll

extern "C" {
ll_status ll_comm_create(const void*, int, int, ll_comm**) {
  ll::set_last_error("NCCL communicator: not built yet");
  return LL_ERR_UNSUPPORTED;
}
ll_status ll_comm_get_unique_id(void*) {
  ll::set_last_error("NCCL communicator: not built yet");
  return LL_ERR_UNSUPPORTED;
}
void ll_comm_destroy(ll_comm*) {}
}
