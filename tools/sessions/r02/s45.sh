# source-level ncu of GAT backward pass A at K=47 (products REUSE layer): hot SASS
M=gpurun_out/s45; mkdir -p $M
B="python bench.py --workload products-gat2-train --steps 1 --warmup 3 --no-e2e --no-regret --no-cpu --no-cold --cuda-graph off"
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"k_gat_bwd_a<.int.8," -s 1 -c 1 -o /tmp/ga $B > $M/ga.log 2>&1; echo "ncu rc=$?"
ncu -i /tmp/ga.ncu-rep --page source --csv --print-source sass > $M/ga_sass.csv 2>/dev/null; echo "src rc=$?"
python tools/sass_hot.py $M/ga_sass.csv > $M/ga_hot.txt; head -60 $M/ga_hot.txt
ncu -i /tmp/ga.ncu-rep --page raw --csv > $M/ga_raw.csv 2>/dev/null
python tools/ncu_summary.py /tmp/ga.ncu-rep > $M/ga_summary.json
