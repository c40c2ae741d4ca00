#!/bin/bash
# ncu --set full of the kernels added late in round 2: the fused pencil pass (sweep2p_kernel<256>, a
# self-exchanged ghost shell on every axis over the peer transport) and the cluster-resident bottom
# (bottom_cluster_kernel, 256^3 L = 4: a 64-brick coarsest level).
cd "${GRAFT_REPO_ROOT:-/root/repo}"
mkdir -p gpurun_out/fin
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
A="--steps 2 --warmup 1 --no-cpu-baseline --no-e2e"
[ -z "$BC" ] && timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"sweep2p_kernel<\(unsigned int\)256>" -s 2 -c 1 \
   -o gpurun_out/fin/prof_peer -f python bench.py $A --ghost-all --transport peer > gpurun_out/fin/ncu_peer.log 2>&1; echo "peer rc=$?"
[ -n "$BC" ] && timeout 900 ncu --set full --clock-control none --import-source on -k regex:bottom_cluster_kernel -s 1 -c 1 \
   -o gpurun_out/fin/prof_bc -f python bench.py $A --n 256 --levels 4 > gpurun_out/fin/ncu_bc.log 2>&1; echo "bc rc=$?"
