M=gpurun_out/s9; mkdir -p $M
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --no-cold"
for w in 1 2 3; do
GRANII_SDDMM_WAVES=$w GRANII_GAT_FUSED=0 timeout 600 $B --workload products-gat2-infer --out $M/gatunf_w$w.json > $M/gatunf_w$w.log 2>&1
GRANII_SDDMM_WAVES=$w timeout 600 $B --workload arxiv-gat-infer --out $M/arxiv_w$w.json > $M/arxiv_w$w.log 2>&1
GRANII_SDDMM_WAVES=$w GRANII_GAT_FUSED=0 timeout 600 $B --workload pubmed-gat2-train --out $M/pubmed_w$w.json > $M/pubmed_w$w.log 2>&1
done
python tools/ab_summary.py $M/*.json
