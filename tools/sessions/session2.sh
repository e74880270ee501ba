# refresh the default-bench evidence for the current kernels: L2 probe, ncu launch list, ncu full (spmm, gemm)
set -u
M=gpurun_out/s2; mkdir -p $M
nvcc -O3 -gencode arch=compute_100a,code=sm_100a tools/probe/l2_bw.cu -o /tmp/l2bw && /tmp/l2bw > $M/l2_peak.json; cat $M/l2_peak.json
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-regret --no-cpu --cuda-graph off"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $M/launches.csv $B > $M/ncu_launch.log 2>&1; echo "ncu launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm_warp -s 20 -c 5 -o $M/spmm_full $B > $M/ncu_spmm.log 2>&1; echo "ncu spmm rc=$?"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:k_gemm -s 4 -c 3 -o $M/gemm_full $B > $M/ncu_gemm.log 2>&1; echo "ncu gemm rc=$?"
for r in spmm_full gemm_full; do [ -f $M/$r.ncu-rep ] && python tools/ncu_summary.py $M/$r.ncu-rep > $M/${r}_summary.json; done
ls -la $M
