# e2e leg with the process bound to the GPU's NUMA node
TAG=${1:-r4h}
cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
cat /sys/bus/pci/devices/*/numa_node 2>/dev/null | sort | uniq -c > gpurun_out/numa_$TAG.txt; lscpu | grep -i numa >> gpurun_out/numa_$TAG.txt 2>&1; nvidia-smi topo -m >> gpurun_out/numa_$TAG.txt 2>&1
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu --no-rho0 --no-traffic > gpurun_out/bench_$TAG.log 2>&1
echo "bench rc=$?" >> gpurun_out/bench_$TAG.log
