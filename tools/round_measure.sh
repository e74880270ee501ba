#!/bin/bash
# one GPU session: calibration, every workload with regret, the regret sweep, the default bench line,
# scaling projections, ncu evidence (writes under gpurun_out/${M:-m})
set -u
M=gpurun_out/${M:-m}
mkdir -p $M
timeout 1500 python -m pytest tests -m gpu -x -q > $M/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -3 $M/pytest_gpu.log
timeout 1500 python tools/calibrate.py --out calib/b200.txt > $M/calib.log 2>&1; echo "calib rc=$?"
cp calib/b200.txt calib/b200_samples.json $M/ 2>/dev/null
for wl in reddit-gcn2-train reddit-gcn2-train-h32 reddit-gcn2-train-h1024 products-gcn2-infer products-gat2-infer products-gat2-train arxiv-gat-infer pubmed-gcn2-train pubmed-gat2-train reddit-sgc-infer reddit-tagcn-infer reddit-gin-infer products-sgc-infer; do
  timeout 600 python bench.py --workload $wl --steps 10 --warmup 3 --no-e2e --no-cpu --out $M/bench_$wl.json > $M/bench_$wl.log 2>&1
  echo "$wl rc=$?"
done
timeout 1500 python tools/regret_sweep.py $M/regret_sweep.json > $M/regret_sweep.log 2>&1; echo "regret sweep rc=$?"
timeout 900 python bench.py --steps 20 --warmup 5 --out $M/bench_default.json > $M/bench_default.log 2>&1; echo "default rc=$?"
[ "${SKIP_NCU:-0}" = 1 ] && { ls $M; exit 0; }
for wl in reddit-gcn2-train products-gcn2-infer products-gat2-infer; do
  timeout 600 python tools/scaling_projection.py --workload $wl --out $M/scaling_projection_$wl.json > $M/proj_$wl.log 2>&1; echo "proj $wl rc=$?"
done
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-regret --no-cpu --cuda-graph off"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $M/launches.csv $B > /dev/null 2>&1; echo "ncu launches rc=$?"
python tools/ncu_launches.py $M/launches.csv $M/ncu_launches_default_bench.txt $M/ncu_launches_share.json "$B" > /dev/null
# full captures stay on the box (/tmp: gpurun copies back <= 64 MiB); summaries come back
R=/tmp/ncu_reps; mkdir -p $R
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm_warp -s 20 -c 5 -o $R/spmm_full $B > /dev/null 2>&1; echo "ncu spmm rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_gemm -s 4 -c 3 -o $R/gemm_full $B > /dev/null 2>&1; echo "ncu gemm rc=$?"
BG="python bench.py --workload products-gat2-train --steps 1 --warmup 3 --no-e2e --no-regret --no-cpu --cuda-graph off"
timeout 900 ncu --set full --clock-control none -k regex:"k_gat_bwd|k_spmm_warp" -s 8 -c 6 -o $R/gat_train_full $BG > /dev/null 2>&1; echo "ncu gat rc=$?"
for r in spmm_full gemm_full gat_train_full; do [ -f $R/$r.ncu-rep ] && python tools/ncu_summary.py $R/$r.ncu-rep > $M/${r}_summary.json; done
[ -f $R/spmm_full.ncu-rep ] && ncu -i $R/spmm_full.ncu-rep --page raw --csv > $M/spmm_full_raw.csv 2>/dev/null
ls $M
