// k_agg_max.cu — instantiations of the aggregation kernel family for M_MAX
// (split per reducer so the templates compile in parallel).
#include "k_agg.cuh"

namespace gnn {
cudaError_t dispatch_max(const KParams &kp, const Mapping &m, int threads, cudaStream_t s) {
  return dispatch_vec<M_MAX>(kp, m, threads, s);
}
}  // namespace gnn
