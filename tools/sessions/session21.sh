set -u
M=gpurun_out/${SESS:-s21}; mkdir -p $M
timeout 1200 python -m pytest tests -m gpu -x -q -k "tagcn or sgc or gat or select or multirank" > $M/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $M/pytest.log
CASES="17:100:256" TUNES="def;16,2,2,4;16,2,2,5;16,2,4,3" timeout 900 python tools/gatbwd_sweep.py products 2>&1 | tail -4
CASES="16:256:47" TUNES="def;8,2,2,4;8,2,2,5;8,2,4,3" timeout 900 python tools/gatbwd_sweep.py products 2>&1 | tail -4
timeout 600 python bench.py --workload reddit-tagcn-infer --steps 5 --warmup 3 --no-e2e --no-cpu --out $M/tagcn.json > $M/tagcn.log 2>&1; echo "tagcn rc=$?"
python -c "import json;d=json.load(open('$M/tagcn.json'));print(d['ms_per_step'],d['config'].get('compositions'),d['per_primitive_ms'],{k:(v.get('regret'),v.get('ms')) for k,v in d.get('selector',{}).items()})"
