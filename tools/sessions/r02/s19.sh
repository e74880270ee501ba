M=gpurun_out/s19; mkdir -p $M
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tn_tc -s 2 -c 2 -o /tmp/tn python bench.py --steps 1 --warmup 3 --no-e2e --no-regret --no-cpu --no-cold --cuda-graph off > $M/ncu.log 2>&1; echo "ncu rc=$?"
python tools/ncu_summary.py /tmp/tn.ncu-rep > $M/tn_summary.json; cat $M/tn_summary.json
ncu -i /tmp/tn.ncu-rep --page raw --csv > $M/tn_raw.csv 2>/dev/null
ncu -i /tmp/tn.ncu-rep --page source --csv > $M/tn_source.csv 2>/dev/null
