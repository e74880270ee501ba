M=gpurun_out/s24; mkdir -p $M
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-regret --no-cpu --no-cold --cuda-graph off"
for wl in reddit-gcn2-train products-gcn2-infer products-gat2-infer products-gat2-train arxiv-gat2-train reddit-gcn2-train-h1024; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none --clock-control none --csv --log-file $M/traffic_$wl.csv $B --workload $wl > $M/traffic_$wl.log 2>&1; echo "$wl rc=$?"
  python tools/ncu_traffic.py $M/traffic_$wl.csv $wl $M/ncu_traffic.json > /dev/null
done
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $M/launches.csv $B > $M/launches.log 2>&1; echo "launches rc=$?"
python tools/ncu_launches.py $M/launches.csv $M/ncu_launches_default_bench.txt $M/ncu_launches_share.json "$B"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_spmm_warp -s 40 -c 2 -o /tmp/rspmm $B > $M/rspmm.log 2>&1; echo "ncu rspmm rc=$?"
python tools/ncu_summary.py /tmp/rspmm.ncu-rep > $M/ncu_reddit_spmm_summary.json
GRANII_GAT_FUSED=0 timeout 900 ncu --set full --clock-control none -k regex:k_sddmm1 -s 4 -c 2 -o /tmp/psddmm $B --workload products-gat2-infer > $M/psddmm.log 2>&1; echo "ncu sddmm rc=$?"
python tools/ncu_summary.py /tmp/psddmm.ncu-rep > $M/ncu_products_sddmm_summary.json
timeout 900 ncu --set full --clock-control none -k regex:k_gemm_tn_tc -s 2 -c 2 -o /tmp/tn $B > $M/tn.log 2>&1; echo "ncu tn rc=$?"
python tools/ncu_summary.py /tmp/tn.ncu-rep > $M/ncu_tn_summary.json
cat $M/ncu_reddit_spmm_summary.json $M/ncu_products_sddmm_summary.json $M/ncu_tn_summary.json | grep -E "kernel|time_ms|dram_read|dram_write|l2_hit|tensor_pct"
