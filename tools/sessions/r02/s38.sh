# R27 check: full-size GAT diag with ambiguous LeakyReLU' rows zeroed, then the full-size tests
M=gpurun_out/s38; mkdir -p $M
timeout 900 python tools/gat_fullsize_diag.py 1 > $M/diag1.log 2>&1; echo "diag1 rc=$?"; head -6 $M/diag1.log
timeout 900 python tools/gat_fullsize_diag.py 0 > $M/diag0.log 2>&1; echo "diag0 rc=$?"; head -5 $M/diag0.log
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -q > $M/pytest_full.log 2>&1; echo "pytest full rc=$?"; tail -3 $M/pytest_full.log; grep "^E  " $M/pytest_full.log | cut -c1-150 | head -4
