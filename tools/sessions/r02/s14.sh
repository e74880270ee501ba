M=gpurun_out/s14; mkdir -p $M
timeout 1200 python -m pytest tests/test_gpu_multirank.py -x -q > $M/pytest_mr.log 2>&1; echo "mr rc=$?"; tail -2 $M/pytest_mr.log
timeout 3000 python tools/regret_sweep.py $M/regret_sweep.json > $M/regret_sweep.log 2>&1; echo "sweep rc=$?"; tail -5 $M/regret_sweep.log
for ph in off 2 3 8; do
  if [ $ph = off ]; then E="GRANII_COMM_OVERLAP=0"; else E="GRANII_COMM_PHASES=$ph"; fi
  env $E timeout 900 python tools/scaling_projection.py --workload products-gcn2-infer --gpus 8 --ranks 0,3,7 --comp 2,3 --out $M/proj_products_$ph.json > $M/proj_products_$ph.log 2>&1; echo "proj $ph rc=$?"; tail -2 $M/proj_products_$ph.log
done
