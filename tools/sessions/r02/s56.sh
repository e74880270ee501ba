# ncu of the update GEMM on products (100 -> 256, 2.45 M rows) and arxiv (64 -> 256 GAT)
M=gpurun_out/s56; mkdir -p $M
B="python bench.py --workload products-gcn2-infer --steps 1 --warmup 2 --no-e2e --no-regret --no-cpu --no-cold --cuda-graph off"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gemm_tc -s 2 -c 2 -o /tmp/pg $B > $M/pg.log 2>&1; echo "ncu pg rc=$?"
python tools/ncu_summary.py /tmp/pg.ncu-rep > $M/pg_summary.json; cat $M/pg_summary.json | grep -E "kernel|time_ms|dram_pct|tensor|issue|warps_active|l2_pct"
ncu -i /tmp/pg.ncu-rep --page raw --csv > $M/pg_raw.csv 2>/dev/null
ncu -i /tmp/pg.ncu-rep --page source --csv --print-source sass > $M/pg_sass.csv 2>/dev/null
B2="python bench.py --workload arxiv-gat-infer --steps 1 --warmup 2 --no-e2e --no-regret --no-cpu --no-cold --cuda-graph off"
timeout 900 ncu --set full --clock-control none -k regex:k_gemm_tc -s 2 -c 2 -o /tmp/ag $B2 > $M/ag.log 2>&1; echo "ncu ag rc=$?"
python tools/ncu_summary.py /tmp/ag.ncu-rep > $M/ag_summary.json; cat $M/ag_summary.json | grep -E "kernel|time_ms|dram_pct|tensor|issue|warps_active|l2_pct"
ncu -i /tmp/ag.ncu-rep --page raw --csv > $M/ag_raw.csv 2>/dev/null
