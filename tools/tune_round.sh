#!/bin/bash
# per-kernel durations of one rank's step (G = 8) with the phased and the all-gather aggregation
O=gpurun_out/tu5; mkdir -p $O
for ph in 2 off; do
  if [ $ph = off ]; then ov=0; unset GRANII_COMM_PHASES; else ov=1; export GRANII_COMM_PHASES=$ph; fi
  timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,lts__t_sector_hit_rate.pct,launch__grid_size --clock-control none --csv --log-file $O/k_$ph.csv \
    python tools/scaling_projection.py --workload products-gcn2-infer --gpus 8 --ranks 0 --steps 1 --warmup 1 --overlap $ov > $O/p_$ph.log 2>&1; echo "$ph rc=$?"
done
unset GRANII_COMM_PHASES
for wl in reddit-gcn2-train:3,3 products-gcn2-infer:2,3; do
  w=${wl%%:*}; c=${wl##*:}
  for ph in 2 3 16 off; do
    if [ $ph = off ]; then ov=0; unset GRANII_COMM_PHASES; else ov=1; export GRANII_COMM_PHASES=$ph; fi
    timeout 300 python tools/scaling_projection.py --workload $w --comp $c --gpus 8 --ranks 0 --overlap $ov --out $O/proj_${w}_$ph.json > $O/proj_${w}_$ph.log 2>&1; echo "$w $ph rc=$?"
  done
done
