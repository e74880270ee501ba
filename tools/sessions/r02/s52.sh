# calibration with the GEMM roofline-time feature, then the regret sweep on it
M=gpurun_out/s52; mkdir -p $M
timeout 1500 python tools/calibrate.py --out $M/b200.txt > $M/calib.log 2>&1; echo "calib rc=$?"; tail -2 $M/calib.log
grep -A1 "gemm" $M/b200.txt
cp $M/b200.txt calib/b200.txt
timeout 1800 python tools/regret_sweep.py $M/regret_sweep.json > $M/regret_sweep.log 2>&1; echo "regret sweep rc=$?"; tail -4 $M/regret_sweep.log
