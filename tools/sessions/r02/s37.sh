# da in fp64 pairs; column-blocked dz / der; parity + full-size + bench
M=gpurun_out/s37; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "gat" > $M/pytest_gat.log 2>&1; echo "pytest gat rc=$?"; tail -2 $M/pytest_gat.log
timeout 900 python bench.py --workload products-gat2-train --steps 10 --warmup 3 --no-cpu --no-e2e --out $M/bench_products-gat2-train.json > $M/bench_pgt.log 2>&1; echo "pgt rc=$?"
python tools/ab_summary.py $M/*.json
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -q -k "products_gat" > $M/pytest_full.log 2>&1; echo "pytest full rc=$?"; tail -3 $M/pytest_full.log; grep "^E  " $M/pytest_full.log | cut -c1-150 | head -4
