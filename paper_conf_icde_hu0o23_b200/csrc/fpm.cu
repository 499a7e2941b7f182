// fpm.cu -- frequent pattern mining (Alg. 2) -- placeholder until the FPM path lands.
#include "internal.cuh"

using namespace gamma_impl;

extern "C" gamma_status gamma_fpm(gamma_graph *g, uint32_t max_edges, uint64_t minsup,
                                  gamma_fpm_result **out) {
  return guarded([&] {
    GAMMA_REQUIRE(g && out, GAMMA_E_INVAL, "gamma_fpm: NULL argument");
    throw Fail{GAMMA_E_UNSUPPORTED, "gamma_fpm: not implemented yet"};
  });
}

extern "C" void gamma_fpm_result_free(gamma_fpm_result *r) {
  if (!r) return;
  delete[] r->pats;
  delete r;
}
