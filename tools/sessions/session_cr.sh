set -u
M=gpurun_out/cr; mkdir -p $M
timeout 900 python -m pytest tests -m gpu -x -q -k "gat" > $M/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $M/pytest_gpu.log
C="python bench.py --workload products-gat2-train --steps 1 --warmup 3 --no-e2e --no-cpu --no-regret --cuda-graph off"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:k_colreduce2 --csv --log-file $M/launches.csv $C > $M/ncu.log 2>&1; echo "ncu rc=$?"
grep -c colreduce2 $M/launches.csv; python - <<'PY'
import csv
rows=[r for r in csv.DictReader(l for l in open('gpurun_out/cr/launches.csv') if l.startswith('"'))]
v=[float(r['Metric Value'].replace(',','')) for r in rows if r.get('Metric Name')=='gpu__time_duration.sum']
print(len(v), sum(v), rows[0].get('Metric Unit') if rows else None, v[:4])
PY
