# NACC accumulators + split cap in the dW GEMM; der-only dz/der passes; full-size parity; benches
M=gpurun_out/s34; mkdir -p $M
timeout 900 python tools/gemm_tn_err.py 0,2048,4096,8192 233000,2449029 > $M/gemm_tn_err.log 2>&1; echo "gemm err rc=$?"; cat $M/gemm_tn_err.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "gemm or gat_recomp_input_layer or gat_backward" > $M/pytest_a.log 2>&1; echo "pytest a rc=$?"; tail -3 $M/pytest_a.log
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -q > $M/pytest_full.log 2>&1; echo "pytest full rc=$?"; tail -3 $M/pytest_full.log
timeout 900 python bench.py --workload products-gat2-train --steps 10 --warmup 3 --no-cpu --out $M/bench_products-gat2-train.json > $M/bench_pgt.log 2>&1; echo "pgt rc=$?"
timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e --out $M/bench_default.json > $M/bench_default.log 2>&1; echo "default rc=$?"
python tools/ab_summary.py $M/*.json
