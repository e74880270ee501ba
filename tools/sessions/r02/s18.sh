M=gpurun_out/s18; mkdir -p $M
for r in 1 0; do GRANII_TN_RAWHI=$r timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "gemm_tn or backward" > $M/pytest_r$r.log 2>&1; echo "rawhi=$r rc=$?"; tail -1 $M/pytest_r$r.log; done
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --no-cold"
for r in 0 1; do for wl in reddit-gcn2-train products-gat2-train; do GRANII_TN_RAWHI=$r timeout 600 $B --workload $wl --out $M/${wl}_r$r.json > $M/${wl}_r$r.log 2>&1; done; done
python tools/ab_summary.py $M/*.json
