#include "internal.h"
namespace atos {
int color_single(atos_csr* g, Part& p, uint64_t seed, int32_t* color_dev, const Resolved& r, atos_stats* st) {
  set_error("colouring not built yet");
  return ATOS_ERR_UNSUPPORTED;
}
}
