// k_agg_att.cu — instantiations of the aggregation kernel family for the
// Table 2 scores other than GAT (NEXT-4, reading R14): Sym-GAT, Linear, GaAN,
// Gene-linear.  One vector per lane (NV = 1); any VEC / LANES.
#include "k_agg.cuh"

namespace gnn {

template <int MODE>
static cudaError_t dispatch_att_mode(const KParams &kp, const Mapping &m, int threads, cudaStream_t s) {
#define GNN_ATT_LANES(V)                                                  \
  switch (m.lanes) {                                                      \
    case 4: return launch_one<MODE, V, 1, 4>(kp, threads, s);             \
    case 8: return launch_one<MODE, V, 1, 8>(kp, threads, s);             \
    case 16: return launch_one<MODE, V, 1, 16>(kp, threads, s);           \
    default: return launch_one<MODE, V, 1, 32>(kp, threads, s);           \
  }
  if (m.nv != 1) return cudaErrorInvalidValue;
  switch (m.vec) {
    case 8: GNN_ATT_LANES(8)
    case 4: GNN_ATT_LANES(4)
    case 2: GNN_ATT_LANES(2)
    default: GNN_ATT_LANES(1)
  }
#undef GNN_ATT_LANES
}

#ifndef GNN_ATT_VECTOR_SCORES
cudaError_t dispatch_att_scalar(const KParams &kp, const Mapping &m, int threads, cudaStream_t s) {
  return kp.mode == M_SYM ? dispatch_att_mode<M_SYM>(kp, m, threads, s) : dispatch_att_mode<M_LIN>(kp, m, threads, s);
}

cudaError_t dispatch_att_vector(const KParams &kp, const Mapping &m, int threads, cudaStream_t s);

cudaError_t dispatch_att(const KParams &kp, const Mapping &m, int threads, cudaStream_t s) {
  return vec_score(kp.mode) ? dispatch_att_vector(kp, m, threads, s) : dispatch_att_scalar(kp, m, threads, s);
}
#else
cudaError_t dispatch_att_vector(const KParams &kp, const Mapping &m, int threads, cudaStream_t s) {
  return kp.mode == M_GAAN ? dispatch_att_mode<M_GAAN>(kp, m, threads, s)
                           : dispatch_att_mode<M_GENE>(kp, m, threads, s);
}
#endif

}  // namespace gnn
