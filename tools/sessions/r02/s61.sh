# repeatability: the regret sweep twice more (model-only 98 / 98 of s52), the default line twice
M=gpurun_out/s61; mkdir -p $M
for i in 1 2; do
  timeout 1800 python tools/regret_sweep.py $M/regret_sweep_$i.json > $M/regret_sweep_$i.log 2>&1; echo "sweep $i rc=$?"; tail -4 $M/regret_sweep_$i.log | head -3
done
for i in 1 2; do
  timeout 900 python bench.py --steps 20 --warmup 5 --no-cpu --out $M/bench_default_$i.json > $M/bench_default_$i.log 2>&1; echo "default $i rc=$?"
done
python tools/ab_summary.py $M/bench_default_*.json
