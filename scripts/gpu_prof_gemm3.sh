# gather roofline microbench + ncu --set full of GEMM3 (the bench's 3rd k_gemm_tc launch)
TAG=${1:-r2}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 ./scripts/gather_roofline > gpurun_out/gather_roofline_$TAG.txt 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tc -s 2 -c 1 -o gpurun_out/prof_gemm3_$TAG -f \
  python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu > gpurun_out/ncu_gemm3_$TAG.log 2>&1
echo "rc=$?" >> gpurun_out/ncu_gemm3_$TAG.log
