#!/bin/bash
# one GPU session: calibration, every workload with regret, the default bench line, ncu evidence
set -u
mkdir -p gpurun_out/m
timeout 900 python tools/calibrate.py --out calib/b200.txt > gpurun_out/m/calib.log 2>&1; cp calib/b200.txt calib/b200_samples.json gpurun_out/m/ 2>/dev/null
for wl in reddit-gcn2-train reddit-gcn2-train-h32 reddit-gcn2-train-h1024 products-gcn2-infer products-gat2-infer arxiv-gat-infer pubmed-gcn2-train; do
  timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 --no-e2e --no-cpu --out gpurun_out/m/bench_$wl.json > gpurun_out/m/bench_$wl.log 2>&1
  echo "$wl rc=$?"
done
timeout 900 python bench.py --steps 20 --warmup 5 --out gpurun_out/m/bench_default.json > gpurun_out/m/bench_default.log 2>&1; echo "default rc=$?"
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-regret --no-cpu --cuda-graph off"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/m/launches.csv $B > /dev/null 2>&1; echo "ncu launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm_warp -s 20 -c 5 -o gpurun_out/m/spmm_full $B > /dev/null 2>&1; echo "ncu spmm rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_gemm -s 4 -c 3 -o gpurun_out/m/gemm_full $B > /dev/null 2>&1; echo "ncu gemm rc=$?"
