M=gpurun_out/s28; mkdir -p $M
for wl in reddit-gcn2-train-h32 reddit-gcn2-train-h1024 products-gcn2-infer products-gat2-infer products-gat2-train arxiv-gat-infer arxiv-gat2-train arxiv-gcn2-train pubmed-gcn2-train pubmed-gat2-train cora-gcn1-infer reddit-sgc-infer reddit-tagcn-infer reddit-gin-infer products-sgc-infer; do
  timeout 900 python bench.py --workload $wl --steps 10 --warmup 3 --no-cpu --out $M/bench_$wl.json > $M/bench_$wl.log 2>&1
  echo "$wl rc=$?"
done
timeout 900 python bench.py --steps 20 --warmup 5 --out $M/bench_default.json > $M/bench_default.log 2>&1; echo "default rc=$?"
timeout 900 python bench.py --impl reference --steps 5 --warmup 3 > $M/bench_reference.log 2>&1; echo "reference rc=$?"; tail -c 600 $M/bench_reference.log
python tools/ab_summary.py $M/*.json
