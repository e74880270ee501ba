# ncu --set full of the gather kernels after the L2 hints: products SDDMM K=1 (+softmax), products SpMM K=100/K=47,
# Reddit SpMM slice, products GAT backward passes
M=gpurun_out/s5; mkdir -p $M; R=/tmp/ncu5; mkdir -p $R
B="python bench.py --steps 1 --warmup 3 --no-e2e --no-regret --no-cpu --no-cold --cuda-graph off"
GRANII_GAT_FUSED=0 timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sddmm1 -s 4 -c 2 -o $R/sddmm $B --workload products-gat2-infer > $M/sddmm.log 2>&1; echo "sddmm rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 4 -c 2 -o $R/pspmm $B --workload products-gcn2-infer > $M/pspmm.log 2>&1; echo "pspmm rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm_warp -s 40 -c 2 -o $R/rspmm $B --workload reddit-gcn2-train > $M/rspmm.log 2>&1; echo "rspmm rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gat_bwd -s 8 -c 4 -o $R/gatbwd $B --workload products-gat2-train > $M/gatbwd.log 2>&1; echo "gatbwd rc=$?"
for r in sddmm pspmm rspmm gatbwd; do
  [ -f $R/$r.ncu-rep ] && python tools/ncu_summary.py $R/$r.ncu-rep > $M/${r}_summary.json
  [ -f $R/$r.ncu-rep ] && ncu -i $R/$r.ncu-rep --page source --csv > $M/${r}_source.csv 2>/dev/null
  [ -f $R/$r.ncu-rep ] && ncu -i $R/$r.ncu-rep --page raw --csv > $M/${r}_raw.csv 2>/dev/null
done
cp $R/sddmm.ncu-rep $M/ 2>/dev/null
ls -la $M
