M=gpurun_out/s11; mkdir -p $M
timeout 300 python tools/sanitize_run.py > $M/plain.log 2>&1; echo "plain rc=$?"; tail -2 $M/plain.log
for tool in memcheck racecheck initcheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 50 python tools/sanitize_run.py > $M/$tool.log 2>&1; echo "$tool rc=$?"; tail -4 $M/$tool.log
done
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --no-cold"
timeout 600 $B --workload cora-gcn1-infer --out $M/cora.json > $M/cora.log 2>&1; echo "cora rc=$?"; tail -c 400 $M/cora.log
timeout 600 $B --workload arxiv-gat2-train --out $M/arxiv_train.json > $M/arxiv_train.log 2>&1; echo "arxiv train rc=$?"
timeout 600 $B --workload arxiv-gcn2-train --out $M/arxiv_gcn_train.json > $M/arxiv_gcn_train.log 2>&1; echo "arxiv gcn train rc=$?"
python tools/ab_summary.py $M/*.json
python -c "import json; d=json.load(open('$M/arxiv_train.json')); print(d['overhead_ms'])"
