// t4_tcgen05.cu — T4: bf16 tcgen05/TMEM contraction (placeholder until the kernel lands).
#include "internal.h"

namespace mdh {

bool t4_supported(const Plan&, std::string* why) {
  if (why) *why = "tcgen05 template not built yet";
  return false;
}
mdh_status prepare_t4(Plan*) { set_error("T4 not available"); return MDH_ERR_UNSUPPORTED; }
mdh_status launch_t4(const Plan&, const void* const*, void* const*, void*, cudaStream_t) {
  set_error("T4 not available");
  return MDH_ERR_UNSUPPORTED;
}
void release_t4(Plan*) {}

}  // namespace mdh
