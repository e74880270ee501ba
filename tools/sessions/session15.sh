set -u
M=gpurun_out/${SESS:-s15}; mkdir -p $M
timeout 900 python -m pytest tests -m gpu -x -q -k "gat" > $M/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $M/pytest.log
CASES="16:64:256;17:64:256" TUNES="def" timeout 900 python tools/gatbwd_sweep.py pubmed 2>&1 | tail -2
for wl in pubmed-gat2-train products-gat2-train; do
  timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 --no-e2e --no-cpu --out $M/bench_$wl.json > $M/bench_$wl.log 2>&1
  echo "$wl rc=$?"
  python -c "import json;d=json.load(open('$M/bench_$wl.json'));print(d['ms_per_step'],d['config'].get('compositions'),d['per_primitive_ms'],{k:(v.get('regret'),v.get('ms'),v.get('selected')) for k,v in d.get('selector',{}).items()})"
done
