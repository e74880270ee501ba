set -u
M=gpurun_out/${SESS:-s37}; mkdir -p $M
timeout 1200 python -m pytest tests -m gpu -x -q -k "gemm or gcn_forward or gat or fullsize or backward" > $M/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $M/pytest.log
python tools/gemm_ab.py split
python tools/gemm_ab.py split
for wl in reddit-gcn2-train products-gcn2-infer products-gat2-infer; do
  timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --no-cold --out $M/bench_$wl.json > $M/bench_$wl.log 2>&1
  python -c "import json;d=json.load(open('$M/bench_$wl.json'));print('$wl', round(d['ms_per_step'],3), {k:round(v,3) for k,v in d['per_primitive_ms'].items()})"
done
