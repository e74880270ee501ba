M=gpurun_out/s20; mkdir -p $M
for bk in 16 32; do GRANII_TN_BK=$bk timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "gemm_tn or backward" > $M/pytest_bk$bk.log 2>&1; echo "bk=$bk rc=$?"; tail -1 $M/pytest_bk$bk.log; done
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --no-cold"
for bk in 32 16; do for wl in reddit-gcn2-train products-gat2-train reddit-gcn2-train-h1024; do GRANII_TN_BK=$bk timeout 600 $B --workload $wl --out $M/${wl}_bk$bk.json > $M/${wl}_bk$bk.log 2>&1; done; done
python tools/ab_summary.py $M/*.json
