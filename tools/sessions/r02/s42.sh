# full measurement of the current tree: GPU tests, calibration, every workload, regret sweep, default line,
# projections, ncu (launch list, DRAM traffic per workload, full captures of the top kernels)
set -u
M=gpurun_out/s42; mkdir -p $M
python -c "import __graft_entry__ as g; g.smoke()" > $M/smoke.log 2>&1; echo "smoke rc=$?"
timeout 1500 python -m pytest tests -m gpu -x -q > $M/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $M/pytest_gpu.log
timeout 1500 python tools/calibrate.py --out $M/b200.txt > $M/calib.log 2>&1; echo "calib rc=$?"; cp calib/b200_samples.json $M/ 2>/dev/null
export GRANII_CALIB=$PWD/$M/b200.txt
for wl in reddit-gcn2-train-h32 reddit-gcn2-train-h1024 products-gcn2-infer products-gat2-infer products-gat2-train arxiv-gat-infer arxiv-gat2-train arxiv-gcn2-train pubmed-gcn2-train pubmed-gat2-train cora-gcn1-infer reddit-sgc-infer reddit-tagcn-infer reddit-gin-infer products-sgc-infer; do
  timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 --no-cpu --out $M/bench_$wl.json > $M/bench_$wl.log 2>&1
  echo "$wl rc=$?"
done
timeout 1800 python tools/regret_sweep.py $M/regret_sweep.json > $M/regret_sweep.log 2>&1; echo "regret sweep rc=$?"; tail -5 $M/regret_sweep.log
timeout 900 python bench.py --steps 20 --warmup 5 --out $M/bench_default.json > $M/bench_default.log 2>&1; echo "default rc=$?"
python tools/ab_summary.py $M/bench_*.json
for wl in reddit-gcn2-train products-gcn2-infer products-gat2-infer; do
  timeout 900 python tools/scaling_projection.py --workload $wl --out $M/scaling_projection_$wl.json > $M/proj_$wl.log 2>&1; echo "proj $wl rc=$?"
done
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-regret --no-cpu --no-cold --cuda-graph off"
for wl in reddit-gcn2-train products-gcn2-infer products-gat2-infer products-gat2-train arxiv-gat2-train reddit-gcn2-train-h1024; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none --clock-control none --csv --log-file $M/traffic_$wl.csv $B --workload $wl > $M/traffic_$wl.log 2>&1; echo "traffic $wl rc=$?"
  python tools/ncu_traffic.py $M/traffic_$wl.csv $wl $M/ncu_traffic.json > /dev/null
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $M/launches.csv $B > $M/launches.log 2>&1; echo "launches rc=$?"
python tools/ncu_launches.py $M/launches.csv $M/ncu_launches_default_bench.txt $M/ncu_launches_share.json "$B"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm_warp -s 40 -c 2 -o /tmp/rspmm $B > $M/rspmm.log 2>&1; echo "ncu rspmm rc=$?"
python tools/ncu_summary.py /tmp/rspmm.ncu-rep > $M/ncu_reddit_spmm_summary.json
timeout 900 ncu --set full --clock-control none -k regex:k_gemm_tn_tc -s 2 -c 2 -o /tmp/tn $B > $M/tn.log 2>&1; echo "ncu tn rc=$?"
python tools/ncu_summary.py /tmp/tn.ncu-rep > $M/ncu_tn_summary.json
timeout 900 ncu --set full --clock-control none -k regex:"k_gat_bwd" -s 4 -c 4 -o /tmp/gat $B --workload products-gat2-train > $M/gat.log 2>&1; echo "ncu gat rc=$?"
python tools/ncu_summary.py /tmp/gat.ncu-rep > $M/ncu_products_gatbwd_summary.json
ls $M | wc -l
