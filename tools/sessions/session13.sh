set -u
M=gpurun_out/${SESS:-s13}; mkdir -p $M
timeout 1500 python -m pytest tests -m gpu -x -q > $M/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $M/pytest_gpu.log
for wl in products-gat2-infer products-gat2-train pubmed-gat2-train arxiv-gat-infer; do
  timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 --no-e2e --no-cpu --out $M/bench_$wl.json > $M/bench_$wl.log 2>&1
  echo "$wl rc=$?"
  python -c "import json;d=json.load(open('$M/bench_$wl.json'));print(d['ms_per_step'],d['config'].get('compositions'),d['per_primitive_ms'],{k:(v.get('regret'),v.get('best'),v.get('selected')) for k,v in d.get('selector',{}).items()})"
done
