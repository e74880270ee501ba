M=gpurun_out/s22; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_multirank.py -x -q -k "gat" > $M/pytest.log 2>&1; echo "pytest rc=$?"; tail -1 $M/pytest.log
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --no-cold"
for h in 0 1 0 1; do GRANII_L2HINT=$h timeout 600 $B --workload products-gat2-train --out $M/pgat_h${h}_$RANDOM.json > /dev/null 2>&1; done
python tools/ab_summary.py $M/*.json
