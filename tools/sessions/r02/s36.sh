# pass A with <dX, Z - P>: accuracy diag, parity, lane-shape sweep on products
M=gpurun_out/s36; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "gat" > $M/pytest_gat.log 2>&1; echo "pytest gat rc=$?"; tail -2 $M/pytest_gat.log
timeout 900 python tools/gat_fullsize_diag.py 0 > $M/diag0.log 2>&1; echo "diag0 rc=$?"; head -4 $M/diag0.log
timeout 900 python tools/gat_fullsize_diag.py 1 > $M/diag1.log 2>&1; echo "diag1 rc=$?"; head -5 $M/diag1.log
CASES="17:100:256:0" TUNES="def;16,2,2,0,1;16,2,2,3,1;4,7,1,0,1;4,7,1,3,1;8,4,1,0,1;8,4,2,0,1;4,8,1,0,1;32,2,1,0,1" timeout 900 python tools/gatbwd_sweep.py products > $M/sweep_recomp.log 2>&1; echo "sweep1 rc=$?"; cat $M/sweep_recomp.log
CASES="16:256:47:1" TUNES="def;8,2,2,0;8,2,2,4;8,2,2,3;4,3,2,0;4,3,4,0;4,3,2,4;4,3,4,3;4,4,2,0" timeout 900 python tools/gatbwd_sweep.py products > $M/sweep_reuse.log 2>&1; echo "sweep2 rc=$?"; cat $M/sweep_reuse.log
