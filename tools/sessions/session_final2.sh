set -u
M=gpurun_out/final2; mkdir -p $M
timeout 900 python bench.py --steps 20 --warmup 5 --out $M/bench_default.json > $M/bench_default.log 2>&1; echo "default rc=$?"; tail -1 $M/bench_default.log | cut -c1-300
C="python bench.py --steps 2 --warmup 3 --no-e2e --no-regret --no-cpu --cuda-graph off"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $M/launches.csv $C > $M/ncu.log 2>&1; echo "ncu rc=$?"
python tools/ncu_launches.py $M/launches.csv $M/ncu_launches_default_bench.txt $M/ncu_launches_share.json "$C"; head -30 $M/ncu_launches_share.json
