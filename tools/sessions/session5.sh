set -u
M=gpurun_out/${SESS:-s5}; mkdir -p $M
timeout 900 python -m pytest tests -m gpu -x -q -k "${KSEL:-sddmm or gat or heavy}" > $M/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $M/pytest.log
for wl in products-gat2-infer arxiv-gat-infer; do
timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --out $M/bench_$wl.json > $M/bench_$wl.log 2>&1; echo "$wl rc=$?"
python -c "import json;d=json.load(open('$M/bench_$wl.json'));print(d['ms_per_step'],d['per_primitive_ms'])"
done
B="python bench.py --workload products-gat2-infer --steps 1 --warmup 3 --no-e2e --no-regret --no-cpu --cuda-graph off"
timeout 600 ncu --set full --clock-control none -k regex:k_sddmm1 -s 6 -c 2 -o $M/sddmm_full $B > $M/ncu_sddmm.log 2>&1; echo "ncu rc=$?"
[ -f $M/sddmm_full.ncu-rep ] && python tools/ncu_summary.py $M/sddmm_full.ncu-rep > $M/sddmm_full_summary.json; cat $M/sddmm_full_summary.json
