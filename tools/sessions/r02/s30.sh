# re-entry check: fresh container rebuild -> GPU tests, default bench, products GAT training line
M=gpurun_out/s30; mkdir -p $M
timeout 1500 python -m pytest tests -m gpu -x -q > $M/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $M/pytest_gpu.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $M/smoke.log 2>&1; echo "smoke rc=$?"
timeout 900 python bench.py --steps 20 --warmup 5 --out $M/bench_default.json > $M/bench_default.log 2>&1; echo "default rc=$?"
timeout 900 python bench.py --workload products-gat2-train --steps 10 --warmup 3 --no-cpu --out $M/bench_products-gat2-train.json > $M/bench_pgt.log 2>&1; echo "pgt rc=$?"
python tools/ab_summary.py $M/*.json
