set -u
M=gpurun_out/${SESS:-s24}; mkdir -p $M
timeout 1200 python -m pytest tests -m gpu -x -q -k "select or gat" > $M/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $M/pytest.log
timeout 1500 python tools/regret_sweep.py $M/regret_sweep.json > $M/regret_sweep.log 2>&1; echo "regret sweep rc=$?"
python -c "import json; d=json.load(open('$M/regret_sweep.json')); print(d['summary'])"
for wl in pubmed-gat2-train arxiv-gat-infer; do
  timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 --no-e2e --no-cpu --out $M/bench_$wl.json > $M/bench_$wl.log 2>&1
  python -c "import json;d=json.load(open('$M/bench_$wl.json'));print('$wl', d['ms_per_step'],d['overhead_ms'],{k:(round(v['regret'],3),v['selected'],round(v['regret_model_only'],3)) for k,v in d['selector'].items()})"
done
