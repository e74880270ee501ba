#!/bin/bash
# ncu --set full of the gather-bound kernels on the products-shaped graph (X > L2): the
# DRAM-bandwidth evidence for SpMM / SDDMM / GAT backward (north_star: >= 60 % of HBM).
set -u
O=gpurun_out/np
mkdir -p $O
B="python bench.py --steps 1 --warmup 3 --no-e2e --no-regret --no-cpu --cuda-graph off"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 6 -c 4 -o $O/gcn_spmm \
  $B --workload products-gcn2-infer > $O/gcn.log 2>&1; echo "gcn rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_spmm|k_sddmm" -s 12 -c 6 -o $O/gat_fwd \
  $B --workload products-gat2-infer > $O/gatf.log 2>&1; echo "gat fwd rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gat_bwd -s 12 -c 4 -o $O/gat_bwd \
  $B --workload products-gat2-train > $O/gatb.log 2>&1; echo "gat bwd rc=$?"
for r in gcn_spmm gat_fwd gat_bwd; do
  [ -f $O/$r.ncu-rep ] && python tools/ncu_summary.py $O/$r.ncu-rep > $O/${r}_summary.json
done
ls -la $O
