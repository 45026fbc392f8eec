// k_agg_att2.cu — the vector-score instantiations (GaAN, Gene-linear) of
// k_agg_att.cu, in their own translation unit so they compile in parallel.
#define GNN_ATT_VECTOR_SCORES
#include "k_agg_att.cu"
