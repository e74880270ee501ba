set -u
M=gpurun_out/elem2; mkdir -p $M
timeout 1500 python -m pytest tests -m gpu -x -q > $M/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $M/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $M/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $M/smoke.log
for wl in products-gat2-train products-gcn2-infer; do
timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --out $M/bench_$wl.json > $M/bench_$wl.log 2>&1; echo "$wl rc=$?"
python -c "import json;d=json.load(open('$M/bench_$wl.json'));print(d['ms_per_step'],d['per_primitive_ms'])"
done
