// k_agg_sum.cu — instantiations of the aggregation kernel family for M_SUM
// (split per reducer so the templates compile in parallel).
#include "k_agg.cuh"

namespace gnn {
cudaError_t dispatch_sum(const KParams &kp, const Mapping &m, int threads, cudaStream_t s) {
  return dispatch_vec<M_SUM>(kp, m, threads, s);
}
}  // namespace gnn
