set -u
M=gpurun_out/s1; mkdir -p $M
nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/probe/l2_bw.cu -o /tmp/l2bw && /tmp/l2bw > $M/l2_peak.json
cat $M/l2_peak.json
timeout 1500 python -m pytest tests -m gpu -x -q > $M/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $M/pytest_gpu.log
timeout 900 python bench.py --steps 20 --warmup 5 --out $M/bench_default.json > $M/bench_default.log 2>&1; echo "default rc=$?"; tail -2 $M/bench_default.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $M/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 $M/smoke.log
