set -u
M=gpurun_out/${SESS:-s14}; mkdir -p $M
B="python bench.py --workload products-gat2-train --steps 1 --warmup 3 --no-e2e --no-regret --no-cpu --cuda-graph off"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $M/launches_gat_train.csv $B > $M/ncu_launch.log 2>&1; echo "ncu launches rc=$?"
python tools/ncu_launches.py $M/launches_gat_train.csv $M/launches_gat_train.txt $M/launches_gat_train_share.json "$B"
CASES="16:64:256;17:64:256;16:32:128;17:128:256" TUNES="def;8,4,2;16,2,2;16,4,2;32,2,1;16,4,1" timeout 900 python tools/gatbwd_sweep.py pubmed > $M/gatbwd_sweep_pubmed.log 2>&1; echo "sweep rc=$?"; cat $M/gatbwd_sweep_pubmed.log
