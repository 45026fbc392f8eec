# DRAM read/write bytes of the three C5 aggregation kernels (write amplification)
# + the per-config report (C1-C4, F sweep) and the C3 ncu DRAM pass on the round-2 graphs
TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python scripts/agg_ab.py warm --once > /dev/null 2>&1  # builds the /tmp graph + plan cache
timeout 900 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,lts__t_sectors_srcunit_tex_op_write.sum,lts__t_sectors_srcunit_tex_aperture_local.sum,l1tex__t_bytes_pipe_lsu_mem_local_op_st.sum,l1tex__t_bytes_pipe_lsu_mem_local_op_ld.sum \
  --clock-control none -k regex:"k_aggregate|k_stream_g4" --csv --log-file gpurun_out/agg_dram_$TAG.csv \
  python scripts/agg_ab.py dram --once > gpurun_out/agg_dram_$TAG.log 2>&1; echo "rc=$?" >> gpurun_out/agg_dram_$TAG.log
bash scripts/gpu_configs.sh $TAG C1,C2,C4,C3,FS
