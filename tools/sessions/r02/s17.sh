M=gpurun_out/s17; mkdir -p $M
GRANII_VBLOCKS=3 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "spmm or gcn or gat or sgc or tagcn or gin or heavy" > $M/pytest_vb3.log 2>&1; echo "vb3 rc=$?"; tail -2 $M/pytest_vb3.log
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --no-cold"
for vb in 1 2 3 4 6 8 12; do
  GRANII_VBLOCKS=$vb timeout 600 $B --workload products-gcn2-infer --out $M/pgcn_vb$vb.json > $M/pgcn_vb$vb.log 2>&1
done
for vb in 1 2 4; do
  GRANII_VBLOCKS=$vb timeout 600 $B --workload reddit-gcn2-train --out $M/reddit_vb$vb.json > $M/reddit_vb$vb.log 2>&1
  GRANII_VBLOCKS=$vb timeout 600 $B --workload arxiv-gcn2-train --out $M/arxiv_vb$vb.json > $M/arxiv_vb$vb.log 2>&1
done
python tools/ab_summary.py $M/*.json
