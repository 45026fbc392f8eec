# GAT register pressure A/B (rows in flight, CTAs per SM) + C3 column-chunk A/B + DRAM write bytes
TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
(timeout 600 python scripts/agg_ab.py default
 for v in GATU3 GATU2 GATMINB3 GATU3MINB3; do GNN_LIB_PATH=$PWD/diag/libgnn_$v.so timeout 300 python scripts/agg_ab.py $v; done
 timeout 300 python scripts/agg_ab.py default) > gpurun_out/agg_ab_$TAG.txt 2>&1
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,l1tex__t_bytes_pipe_lsu_mem_local_op_st.sum,l1tex__t_bytes_pipe_lsu_mem_local_op_ld.sum \
  --clock-control none -k regex:"k_aggregate|k_stream_g4" --csv --log-file gpurun_out/agg_dram_$TAG.csv \
  python scripts/agg_ab.py dram --once > gpurun_out/agg_dram_$TAG.log 2>&1
timeout 900 python scripts/c3_chunk.py C3 > gpurun_out/c3_chunk_$TAG.txt 2>&1
