# der-only RECOMP input-layer backward: parity, full-size products GAT training, bench
M=gpurun_out/s31; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "gat_recomp_input_layer or gat_backward" > $M/pytest_gat.log 2>&1; echo "pytest gat rc=$?"; tail -3 $M/pytest_gat.log
timeout 900 python -m pytest tests/test_gpu_fullsize.py -q -k "products_gat_training" > $M/pytest_full.log 2>&1; echo "pytest full rc=$?"; tail -3 $M/pytest_full.log
timeout 900 python bench.py --workload products-gat2-train --steps 10 --warmup 3 --no-cpu --out $M/bench_products-gat2-train.json > $M/bench_pgt.log 2>&1; echo "pgt rc=$?"
python tools/ab_summary.py $M/*.json
