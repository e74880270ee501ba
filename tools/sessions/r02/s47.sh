# final-tree measurement: smoke, GPU suite, every workload's line, regret sweep (refine up to 10 ms), default line
set -u
M=gpurun_out/s47; mkdir -p $M
python -c "import __graft_entry__ as g; g.smoke()" > $M/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $M/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > $M/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $M/pytest_gpu.log; grep -E "^E " $M/pytest_gpu.log | head -5
for wl in reddit-gcn2-train-h32 reddit-gcn2-train-h1024 products-gcn2-infer products-gat2-infer products-gat2-train arxiv-gat-infer arxiv-gat2-train arxiv-gcn2-train pubmed-gcn2-train pubmed-gat2-train cora-gcn1-infer reddit-sgc-infer reddit-tagcn-infer reddit-gin-infer products-sgc-infer; do
  timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 --no-cpu --out $M/bench_$wl.json > $M/bench_$wl.log 2>&1
  echo "$wl rc=$?"
done
timeout 1800 python tools/regret_sweep.py $M/regret_sweep.json > $M/regret_sweep.log 2>&1; echo "regret sweep rc=$?"; tail -4 $M/regret_sweep.log
timeout 900 python bench.py --steps 20 --warmup 5 --out $M/bench_default.json > $M/bench_default.log 2>&1; echo "default rc=$?"
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > $M/bench_reference.log 2>&1; echo "reference rc=$?"; tail -1 $M/bench_reference.log | cut -c1-400
python tools/ab_summary.py $M/bench_*.json
