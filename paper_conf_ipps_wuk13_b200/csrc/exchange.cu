// exchange.cu — multi-GPU exchange (placeholder until the NCCL / loopback
// backends land; world == 1 never reaches this file).
#include "exchange.h"

namespace sg {

struct Exchange {
  int dummy = 0;
};

[[noreturn]] static void not_yet(sg_graph *g, const char *what) {
  fail(g, SG_EINVAL, std::string(what) + ": multi-GPU exchange not available in this build");
}

Exchange *exchange_create(sg_graph *g, const sg_dist *) { not_yet(g, "create"); }
void exchange_destroy(Exchange *x) { delete x; }
void exchange_row_counts(sg_graph *g, int, int64_t) { not_yet(g, "pass"); }
void exchange_and_group(sg_graph *g, int) { not_yet(g, "group"); }
int64_t exchange_sum(sg_graph *g, int64_t) { not_yet(g, "counts"); }
void exchange_require_single(sg_graph *g, const char *what) { not_yet(g, what); }

}  // namespace sg

struct sg_loopback {
  int world;
};

extern "C" sg_status sg_loopback_create(int32_t world, sg_loopback **out) {
  if (!out || world < 1) return SG_EINVAL;
  *out = new sg_loopback{world};
  return SG_OK;
}

extern "C" void sg_loopback_destroy(sg_loopback *lb) { delete lb; }
