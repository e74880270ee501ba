M=gpurun_out/s13; mkdir -p $M
timeout 2400 python tools/calibrate.py --out calib/b200.txt > $M/calib.log 2>&1; echo "calib rc=$?"; tail -30 $M/calib.log
cp calib/b200.txt calib/b200_samples.json $M/ 2>/dev/null
timeout 3000 python tools/regret_sweep.py $M/regret_sweep.json > $M/regret_sweep.log 2>&1; echo "sweep rc=$?"; tail -8 $M/regret_sweep.log
