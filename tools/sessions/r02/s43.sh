# pipelined entry-tile SDDMM + SpMM 8x3 shape (32 < K <= 48): parity, A/B timings; GAT backward K=47 shape sweep;
# regret sweep with the refit calibration
M=gpurun_out/s43; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "sddmm or heavy_row or spmm or gat_forward or gat_fused" > $M/pytest_a.log 2>&1; echo "pytest a rc=$?"; tail -2 $M/pytest_a.log; grep -E "^E " $M/pytest_a.log | head -5
timeout 900 python -m pytest tests/test_gpu_multirank.py -q -x -k "gat_forward_backward" > $M/pytest_b.log 2>&1; echo "pytest b rc=$?"; tail -2 $M/pytest_b.log; grep -E "^E " $M/pytest_b.log | head -5
timeout 300 python tools/sddmm_tile_ab.py pubmed,arxiv,reddit,products 1 > $M/sddmm_pipe.log 2>&1; cat $M/sddmm_pipe.log
for K in 0 1; do
  GRANII_SPMM_K48=$K timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --out $M/default_k48_$K.json > /dev/null 2>&1; echo "default k48=$K rc=$?"
  GRANII_SPMM_K48=$K timeout 600 python bench.py --workload products-gcn2-infer --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --out $M/pgcn_k48_$K.json > /dev/null 2>&1; echo "pgcn k48=$K rc=$?"
  GRANII_SPMM_K48=$K timeout 600 python bench.py --workload products-gat2-infer --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --out $M/pgat_k48_$K.json > /dev/null 2>&1; echo "pgat k48=$K rc=$?"
done
python tools/ab_summary.py $M/*_k48_*.json
CASES="16:256:47:1" TUNES="def;4,3,2,0;4,3,4,0;4,3,2,4;4,3,4,3;4,4,2,0;8,2,2,4" timeout 900 python tools/gatbwd_sweep.py products > $M/sweep_k47.log 2>&1; echo "sweep rc=$?"; cat $M/sweep_k47.log
timeout 1800 python tools/regret_sweep.py $M/regret_sweep.json > $M/regret_sweep.log 2>&1; echo "regret sweep rc=$?"; tail -4 $M/regret_sweep.log
