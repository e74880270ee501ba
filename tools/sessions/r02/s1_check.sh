set -u
M=gpurun_out/s1; mkdir -p $M
python -c "import __graft_entry__ as g; g.smoke()" > $M/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1800 python -m pytest tests -m gpu -x -q > $M/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $M/pytest_gpu.log
timeout 900 python bench.py --steps 20 --warmup 5 --out $M/bench_default.json > $M/bench_default.log 2>&1; echo "default rc=$?"
timeout 600 python bench.py --workload products-gat2-train --steps 10 --warmup 3 --no-e2e --no-cpu --out $M/bench_pgat.json > $M/bench_pgat.log 2>&1; echo "pgat rc=$?"
