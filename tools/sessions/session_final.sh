set -u
M=gpurun_out/final; mkdir -p $M
timeout 1500 python -m pytest tests -m gpu -x -q > $M/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $M/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $M/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 $M/smoke.log
timeout 900 python bench.py --steps 20 --warmup 5 --out $M/bench_default.json > $M/bench_default.log 2>&1; echo "default rc=$?"; tail -2 $M/bench_default.log
timeout 600 python bench.py --impl reference --steps 2 --warmup 3 > $M/bench_ref.log 2>&1; echo "ref rc=$?"; tail -1 $M/bench_ref.log
