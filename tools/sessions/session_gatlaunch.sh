set -u
M=gpurun_out/gl; mkdir -p $M
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $M/launches.csv python bench.py --workload products-gat2-train --steps 1 --warmup 3 --no-e2e --no-cpu --no-regret --cuda-graph off > $M/b.log 2>&1; echo "ncu rc=$?"
python - <<'PY'
import csv, collections
rows=[r for r in csv.DictReader(l for l in open('gpurun_out/gl/launches.csv') if l.startswith('"'))]
t=collections.defaultdict(float); n=collections.Counter()
for r in rows:
    if r.get('Metric Name')=='gpu__time_duration.sum':
        k=r['Kernel Name'][:90]; v=float(r['Metric Value'].replace(',',''))
        u=r.get('Metric Unit','')
        v = v/1e6 if u=='ns' else (v/1e3 if u in ('us','usecond') else v)
        t[k]+=v; n[k]+=1
for k,v in sorted(t.items(), key=lambda x:-x[1])[:30]: print(f"{v:10.3f} ms {n[k]:5d}  {k}")
PY
