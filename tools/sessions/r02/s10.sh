M=gpurun_out/s10; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -x -q -k "sddmm or spmm or gat or heavy or gcn or directed" > $M/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $M/pytest.log
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --no-cold"
GRANII_GAT_FUSED=0 timeout 600 $B --workload products-gat2-infer --out $M/gatunf.json > $M/gatunf.log 2>&1
for wl in arxiv-gat-infer reddit-gcn2-train products-gcn2-infer products-gat2-infer pubmed-gcn2-train products-gat2-train; do
  timeout 600 $B --workload $wl --out $M/${wl}.json > $M/${wl}.log 2>&1
done
python tools/ab_summary.py $M/*.json
