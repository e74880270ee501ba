M=gpurun_out/s4; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "spmm or sddmm or gat_fused or heavy" > $M/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $M/pytest.log
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --no-cold"
for wl in reddit-gcn2-train products-gcn2-infer products-gat2-train; do
  for h in 0 1; do
    GRANII_L2HINT=$h timeout 600 $B --workload $wl --out $M/${wl}_h$h.json > $M/${wl}_h$h.log 2>&1
  done
done
for h in 0 1; do GRANII_GAT_FUSED=0 GRANII_L2HINT=$h timeout 600 $B --workload products-gat2-infer --out $M/gatunf_h$h.json > $M/gatunf_h$h.log 2>&1; done
python tools/ab_summary.py $M/*.json
