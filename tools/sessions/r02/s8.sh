M=gpurun_out/s8; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "sddmm or spmm or gat_fused or heavy or gcn_forward" > $M/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $M/pytest.log
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --no-cold"
GRANII_GAT_FUSED=0 timeout 600 $B --workload products-gat2-infer --out $M/gatunf.json > $M/gatunf.log 2>&1
timeout 600 $B --workload arxiv-gat-infer --out $M/arxiv.json > $M/arxiv.log 2>&1
for w in 0 1; do
  for wl in reddit-gcn2-train products-gcn2-infer products-gat2-infer pubmed-gcn2-train; do
    GRANII_SPMM_WAVES=$w timeout 600 $B --workload $wl --out $M/${wl}_w$w.json > $M/${wl}_w$w.log 2>&1
  done
done
python tools/ab_summary.py $M/*.json
