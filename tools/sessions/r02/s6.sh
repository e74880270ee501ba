M=gpurun_out/s6; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -x -q -k "sddmm or gat or gcn_forward or heavy or directed" > $M/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $M/pytest.log
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --no-cold"
for o in 0 1; do GRANII_SDDMM_ORDERED=$o GRANII_GAT_FUSED=0 timeout 600 $B --workload products-gat2-infer --out $M/gatunf_o$o.json > $M/gatunf_o$o.log 2>&1; done
for o in 0 1; do GRANII_SDDMM_ORDERED=$o timeout 600 $B --workload arxiv-gat-infer --out $M/arxiv_o$o.json > $M/arxiv_o$o.log 2>&1; done
for o in 0 1; do GRANII_SDDMM_ORDERED=$o timeout 600 $B --workload pubmed-gat2-train --out $M/pubmedgat_o$o.json > $M/pubmedgat_o$o.log 2>&1; done
python tools/ab_summary.py $M/*.json
GRANII_GAT_FUSED=0 timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_sddmm1 -s 4 -c 2 -o /tmp/sddmm_blk python bench.py --steps 1 --warmup 3 --no-e2e --no-regret --no-cpu --no-cold --cuda-graph off --workload products-gat2-infer > $M/ncu.log 2>&1; echo "ncu rc=$?"
python tools/ncu_summary.py /tmp/sddmm_blk.ncu-rep > $M/sddmm_blk_summary.json; cat $M/sddmm_blk_summary.json | head -40
ncu -i /tmp/sddmm_blk.ncu-rep --page source --csv > $M/sddmm_blk_source.csv 2>/dev/null
