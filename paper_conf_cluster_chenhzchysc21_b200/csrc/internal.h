// internal.h — host-side internals shared by api.cu and select.cpp.
#pragma once
#include <cstdint>
#include <vector>

#include "../../include/cswap.h"

namespace cswap {

struct ProbeEstimates {
  uint64_t zeros, nnz, runs, zero_runs;
};

ProbeEstimates estimate(uint64_t n, const cswap_probe_result& p);
void decide(uint64_t n, int w, const cswap_probe_result& p, double hidden_f, double hidden_b, const cswap_calib& c,
            cswap_decision* out);
bool fit3(const double* S, const double* s, const double* t, uint64_t m, double* beta);
bool fit_general(const double* X, const double* y, uint64_t m, uint32_t p, double* beta);
bool fit_link(const double* bytes, const double* t, uint64_t m, double* alpha, double* bw);
void default_calib(cswap_calib* c);

}  // namespace cswap
