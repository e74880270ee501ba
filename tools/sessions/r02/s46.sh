# GAT backward: 32-bit masks + IMAD.WIDE.U32 row addresses -- parity, products training, hot-loop instruction count
M=gpurun_out/s46; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "gat" > $M/pytest_gat.log 2>&1; echo "pytest gat rc=$?"; tail -2 $M/pytest_gat.log; grep -E "^E " $M/pytest_gat.log | head -5
timeout 900 python -m pytest tests/test_gpu_multirank.py -q -x -k "gat" > $M/pytest_mr.log 2>&1; echo "pytest mr rc=$?"; tail -2 $M/pytest_mr.log
timeout 600 python bench.py --workload products-gat2-train --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --out $M/pgt.json > /dev/null 2>&1; echo "pgt rc=$?"
timeout 600 python bench.py --workload arxiv-gat2-train --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --out $M/agt.json > /dev/null 2>&1; echo "agt rc=$?"
timeout 600 python bench.py --workload pubmed-gat2-train --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --out $M/pubgt.json > /dev/null 2>&1; echo "pubgt rc=$?"
python tools/ab_summary.py $M/*.json
B="python bench.py --workload products-gat2-train --steps 1 --warmup 3 --no-e2e --no-regret --no-cpu --no-cold --cuda-graph off"
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"k_gat_bwd_(a|b)<.int.8," -s 2 -c 2 -o /tmp/ga $B > $M/ga.log 2>&1; echo "ncu rc=$?"
ncu -i /tmp/ga.ncu-rep --page source --csv --print-source sass > $M/ga_sass.csv 2>/dev/null
python tools/ncu_summary.py /tmp/ga.ncu-rep > $M/ga_summary.json; cat $M/ga_summary.json | grep -E "kernel|time_ms|dram_pct|inst_M|issue"
