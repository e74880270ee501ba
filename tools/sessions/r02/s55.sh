# final-tree measurement after the recalibration and the GAT reductions: smoke, GPU suite, every workload's line,
# default line (e2e + CPU baseline), reference arm, projections, launch list + DRAM traffic of the changed paths
set -u
M=gpurun_out/s55; mkdir -p $M
python -c "import __graft_entry__ as g; g.smoke()" > $M/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $M/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > $M/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $M/pytest_gpu.log; grep -E "^E " $M/pytest_gpu.log | head -5
for wl in reddit-gcn2-train-h32 reddit-gcn2-train-h1024 products-gcn2-infer products-gat2-infer products-gat2-train arxiv-gat-infer arxiv-gat2-train arxiv-gcn2-train pubmed-gcn2-train pubmed-gat2-train cora-gcn1-infer reddit-sgc-infer reddit-tagcn-infer reddit-gin-infer products-sgc-infer; do
  timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 --no-cpu --out $M/bench_$wl.json > $M/bench_$wl.log 2>&1
  echo "$wl rc=$?"
done
timeout 900 python bench.py --steps 20 --warmup 5 --out $M/bench_default.json > $M/bench_default.log 2>&1; echo "default rc=$?"
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > $M/bench_reference.log 2>&1; echo "reference rc=$?"
python tools/ab_summary.py $M/bench_*.json
for wl in reddit-gcn2-train products-gcn2-infer products-gat2-infer; do
  timeout 900 python tools/scaling_projection.py --workload $wl --out $M/scaling_projection_$wl.json > $M/proj_$wl.log 2>&1; echo "proj $wl rc=$?"
done
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-regret --no-cpu --no-cold --cuda-graph off"
for wl in products-gat2-train arxiv-gat2-train; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none --clock-control none --csv --log-file $M/traffic_$wl.csv $B --workload $wl > $M/traffic_$wl.log 2>&1; echo "traffic $wl rc=$?"
  python tools/ncu_traffic.py $M/traffic_$wl.csv $wl $M/ncu_traffic.json > /dev/null
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $M/launches.csv $B > $M/launches.log 2>&1; echo "launches rc=$?"
python tools/ncu_launches.py $M/launches.csv $M/ncu_launches_default_bench.txt $M/ncu_launches_share.json "$B" > /dev/null
