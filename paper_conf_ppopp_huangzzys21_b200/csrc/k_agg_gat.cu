// k_agg_gat.cu — instantiations of the aggregation kernel family for M_GAT
// (split per reducer so the templates compile in parallel).
#include "k_agg.cuh"

namespace gnn {
cudaError_t dispatch_gat(const KParams &kp, const Mapping &m, int threads, cudaStream_t s) {
  return dispatch_vec<M_GAT>(kp, m, threads, s);
}
}  // namespace gnn
