# full-size products SDDMM (entry tiles) parity; empty-graph SDDMM; the SDDMM / multirank GAT tests
M=gpurun_out/s49; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "sddmm" > $M/pytest_a.log 2>&1; echo "pytest a rc=$?"; tail -2 $M/pytest_a.log; grep -E "^E " $M/pytest_a.log | head -5
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -q -x -k "sddmm" > $M/pytest_full.log 2>&1; echo "pytest full rc=$?"; tail -2 $M/pytest_full.log; grep -E "^E " $M/pytest_full.log | head -8
