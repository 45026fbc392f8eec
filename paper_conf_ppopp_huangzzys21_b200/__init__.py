"""paper_conf_ppopp_huangzzys21_b200 — B200-native (sm_100a) GNN neighbor aggregation.

The hot path of Huang et al., "Understanding and Bridging the Gaps in Current
GNN Performance Optimizations" (PPoPP'21): CSR graph operations (sum / mean /
max), the fused GAT edge-softmax aggregation, EdgeConv max aggregation, the
X.W transform, locality-aware task scheduling and neighbor grouping.

The product is ``libgnn.so`` (C-ABI, ``include/gnn.h``); ``gnn`` is its thin
Python binding.  Touching any public name loads the library and fails loudly
if it is not built — there is no CPU fallback.  (The submodule ``build`` can
be imported without loading the library, so it can rebuild it.)
"""
_PUBLIC = ("Plan", "aggregate", "aggregate_accumulate", "scale_rows", "gat_aggregate", "gat_layer", "gat_transform", "edgeconv", "edgeconv_aggregate", "gemm", "gemm_mirrored", "IpcBuffer", "ipc_open", "ipc_close",
           "gcn_layer", "partition_rows", "local_csr", "local_csr_block", "launch_count", "set_gemm_impl", "set_agg_mapping", "set_group_size", "tune_aggregate", "attn_aggregate", "sample_neighbors", "sage_lstm_aggregate", "sage_lstm_layer", "las_host", "groups_host",
           "GnnError")
__all__ = ["gnn", *_PUBLIC]


def __getattr__(name):
    if name == "gnn" or name in _PUBLIC:
        import importlib
        _gnn = importlib.import_module(__name__ + ".gnn")
        return _gnn if name == "gnn" else getattr(_gnn, name)
    raise AttributeError(name)
