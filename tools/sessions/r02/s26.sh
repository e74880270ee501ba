M=gpurun_out/s26; mkdir -p $M
for n in 8 4; do GRANII_TN_NCW=$n timeout 600 python -m pytest tests/test_gpu_parity.py -x -q -k "gemm_tn or gcn_backward" > $M/pytest_n$n.log 2>&1; echo "ncw=$n rc=$?"; tail -1 $M/pytest_n$n.log; done
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --no-cold"
for n in 4 8 4 8; do for wl in reddit-gcn2-train products-gat2-train; do GRANII_TN_NCW=$n timeout 600 $B --workload $wl --out $M/${wl}_n${n}_$RANDOM.json > /dev/null 2>&1; done; done
python tools/ab_summary.py $M/*.json
