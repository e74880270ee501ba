# per-kernel launch list of the arxiv / products GAT training steps (elementwise share)
M=gpurun_out/s53; mkdir -p $M
for wl in arxiv-gat2-train products-gat2-train; do
B="python bench.py --workload $wl --steps 1 --warmup 3 --no-e2e --no-regret --no-cpu --no-cold --cuda-graph off"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $M/launches_$wl.csv $B > $M/launches_$wl.log 2>&1; echo "launches $wl rc=$?"
python tools/ncu_launches.py $M/launches_$wl.csv $M/launches_$wl.txt $M/share_$wl.json "$B" > /dev/null
python -c "
import json; d=json.load(open('$M/share_$wl.json'))
for k,v in sorted(d.items(), key=lambda x:-x[1]['us'])[:14]: print(round(v['us'],1), v['launches'], k[:110])
"
done
