// match.cu -- subgraph matching (Alg. 1) -- placeholder until the SM path lands.
#include "internal.cuh"

using namespace gamma_impl;

extern "C" gamma_status gamma_match(gamma_graph *g, const gamma_pattern *p, uint64_t *count,
                                    uint64_t *mappings) {
  return guarded([&] {
    GAMMA_REQUIRE(g && p && count, GAMMA_E_INVAL, "gamma_match: NULL argument");
    throw Fail{GAMMA_E_UNSUPPORTED, "gamma_match: not implemented yet"};
  });
}

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
