# experiment: 128-byte-aligned rows (ld 64) for the K = 41 / 47 internal buffers
M=gpurun_out/s48; mkdir -p $M
for L in 0 1 0 1; do
  GRANII_LD_LINE=$L timeout 600 python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --out $M/default_ld$L.json > /dev/null 2>&1; echo "default ld=$L rc=$?"; python tools/ab_summary.py $M/default_ld$L.json
done
for L in 0 1; do
  GRANII_LD_LINE=$L timeout 600 python bench.py --workload products-gcn2-infer --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --out $M/pgcn_ld$L.json > /dev/null 2>&1; echo "pgcn ld=$L rc=$?"
done
python tools/ab_summary.py $M/pgcn_ld*.json
GRANII_LD_LINE=1 timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "gcn_forward or gcn_backward" > $M/pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $M/pytest.log
