# GAT backward small reductions (colreduce2 vectorised, sum_chunks warp per output, mattvec2 row groups): parity + timing
M=gpurun_out/s54; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "gat" > $M/pytest_gat.log 2>&1; echo "pytest gat rc=$?"; tail -2 $M/pytest_gat.log; grep -E "^E " $M/pytest_gat.log | head -5
timeout 900 python -m pytest tests/test_gpu_multirank.py -q -x -k "gat" > $M/pytest_mr.log 2>&1; echo "pytest mr rc=$?"; tail -2 $M/pytest_mr.log
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -q -x -k "products_gat" > $M/pytest_full.log 2>&1; echo "pytest full rc=$?"; tail -2 $M/pytest_full.log; grep -E "^E " $M/pytest_full.log | head -5
for wl in arxiv-gat2-train pubmed-gat2-train products-gat2-train; do
timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --out $M/$wl.json > /dev/null 2>&1; echo "$wl rc=$?"
done
python tools/ab_summary.py $M/*.json
B="python bench.py --workload arxiv-gat2-train --steps 1 --warmup 3 --no-e2e --no-regret --no-cpu --no-cold --cuda-graph off"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $M/launches.csv $B > /dev/null 2>&1
python tools/ncu_launches.py $M/launches.csv $M/launches.txt $M/share.json "$B" > /dev/null
grep -E "colreduce|mattvec|sum_chunks" $M/launches.txt | head -12
