// pf_tuned.cu -- tuned sweeps (placeholder: routes to the naive kernels until
// the z-marching kernels land).
#include "pf_model.cuh"

namespace pf {
void launch_tuned_phi(const DevParams& P, const Geom& g, const Tables& T, const double* ps, const double* ms,
                      double* pd, cudaStream_t s) {
  launch_phi_naive(P, g, T, ps, ms, pd, s);
}
void launch_tuned_mu(const DevParams& P, const Geom& g, const Tables& T, const double* ps, const double* pd,
                     const double* ms, double* md, cudaStream_t s) {
  launch_mu_naive(P, g, T, ps, pd, ms, md, s);
}
}  // namespace pf
