# products GAT: dz hub segments, bench; full-size error diagnosis (both layers)
M=gpurun_out/s35; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "gat_recomp_input_layer" > $M/pytest_a.log 2>&1; echo "pytest a rc=$?"; tail -2 $M/pytest_a.log
timeout 900 python bench.py --workload products-gat2-train --steps 10 --warmup 3 --no-cpu --no-e2e --out $M/bench_products-gat2-train.json > $M/bench_pgt.log 2>&1; echo "pgt rc=$?"
python tools/ab_summary.py $M/*.json
timeout 900 python tools/gat_fullsize_diag.py 1 > $M/diag1.log 2>&1; echo "diag1 rc=$?"; cat $M/diag1.log
timeout 900 python tools/gat_fullsize_diag.py 0 > $M/diag0.log 2>&1; echo "diag0 rc=$?"; cat $M/diag0.log
