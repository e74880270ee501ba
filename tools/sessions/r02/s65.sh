# experiment: fewer, longer dW splits on small graphs (GRANII_TN_MIN_KB: k-blocks per split, no wave rounding)
M=gpurun_out/s65; mkdir -p $M
for wl in arxiv-gcn2-train pubmed-gcn2-train arxiv-gat2-train; do
  for KB in def 32 64 128; do
    if [ $KB = def ]; then unset GRANII_TN_MIN_KB; else export GRANII_TN_MIN_KB=$KB; fi
    timeout 600 python bench.py --workload $wl --steps 20 --warmup 5 --no-e2e --no-cpu --no-regret --out $M/${wl}_$KB.json > /dev/null 2>&1; echo "$wl $KB rc=$?"
  done
  unset GRANII_TN_MIN_KB
done
python tools/ab_summary.py $M/*.json
