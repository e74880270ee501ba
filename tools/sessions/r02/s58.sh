# entry-tile SDDMM with dynamically distributed rows: parity + A/B
M=gpurun_out/s58; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "sddmm" > $M/pytest_a.log 2>&1; echo "pytest a rc=$?"; tail -2 $M/pytest_a.log; grep -E "^E " $M/pytest_a.log | head -5
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -q -x -k "sddmm" > $M/pytest_full.log 2>&1; echo "pytest full rc=$?"; tail -1 $M/pytest_full.log
timeout 900 python -m pytest tests/test_gpu_multirank.py -q -x -k "gat_forward_backward" > $M/pytest_mr.log 2>&1; echo "pytest mr rc=$?"; tail -1 $M/pytest_mr.log
timeout 300 python tools/sddmm_tile_ab.py pubmed,arxiv,reddit,products > $M/ab.log 2>&1; cat $M/ab.log
