// dist.cu — multi-GPU sharding.  Placeholder until the NCCL exchange lands:
// distributed handles report SESA_ENCCL.
#include "sesa_internal.h"

struct DistState {};

sesa_status sesa_trace::check_dist(const sesa_access*, uint64_t, uint64_t) {
  fail(SESA_ENCCL, "distributed race check not available in this build");
  return status;
}

void sesa_trace::destroy_dist() {}

extern "C" {
sesa_status sesa_trace_create_dist(const sesa_config*, int, int, const uint8_t*, sesa_trace** out) {
  if (out) *out = nullptr;
  return SESA_ENCCL;
}
sesa_status sesa_nccl_unique_id(uint8_t*) { return SESA_ENCCL; }
}
