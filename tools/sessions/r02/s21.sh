M=gpurun_out/s21; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "spmm or gat or gcn" > $M/pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $M/pytest.log
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --no-cold"
for p in 0 1; do for wl in products-gcn2-infer products-gat2-train products-gat2-infer reddit-gcn2-train arxiv-gat2-train; do GRANII_PREFETCH=$p timeout 600 $B --workload $wl --out $M/${wl}_p$p.json > $M/${wl}_p$p.log 2>&1; done; done
python tools/ab_summary.py $M/*.json
