set -u
M=gpurun_out/${SESS:-s29}; mkdir -p $M; R=/tmp/reps; mkdir -p $R
B="python bench.py --workload products-gcn2-infer --steps 1 --warmup 2 --no-e2e --no-regret --no-cpu --no-cold --cuda-graph off"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tc -s 2 -c 2 -o $R/pgemm $B > $M/ncu.log 2>&1; echo "ncu rc=$?"
python tools/ncu_summary.py $R/pgemm.ncu-rep > $M/pgemm_summary.json
ncu -i $R/pgemm.ncu-rep --page source --csv --print-source sass > $M/pgemm_src.csv 2>/dev/null
ncu -i $R/pgemm.ncu-rep --page raw --csv > $M/pgemm_raw.csv 2>/dev/null
ncu -i $R/pgemm.ncu-rep --page details --csv > $M/pgemm_details.csv 2>/dev/null
ls -la $M
