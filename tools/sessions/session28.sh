set -u
M=gpurun_out/s28; mkdir -p $M; R=/tmp/reps; mkdir -p $R
B="python bench.py --workload products-gcn2-infer --steps 1 --warmup 2 --no-e2e --no-regret --no-cpu --no-cold --cuda-graph off"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm_warp -s 2 -c 2 -o $R/pspmm $B > $M/ncu.log 2>&1; echo "ncu rc=$?"
python tools/ncu_summary.py $R/pspmm.ncu-rep > $M/pspmm_summary.json
ncu -i $R/pspmm.ncu-rep --page source --csv --print-source sass > $M/pspmm_src.csv 2>/dev/null
ncu -i $R/pspmm.ncu-rep --page raw --csv > $M/pspmm_raw.csv 2>/dev/null
ls -la $M
