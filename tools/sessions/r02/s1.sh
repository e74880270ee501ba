M=gpurun_out/s1; mkdir -p $M
nproc > $M/host.txt; free -g >> $M/host.txt
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q -k "refine or misaligned or gat_backward_both" > $M/pytest_new.log 2>&1; echo "new rc=$?"; tail -3 $M/pytest_new.log
timeout 2400 python -m pytest tests/test_gpu_fullsize.py -x -q --durations=10 > $M/pytest_full.log 2>&1; echo "full rc=$?"; tail -15 $M/pytest_full.log
