# entry-tile K=1 SDDMM: parity (new tile tests + the SDDMM / GAT tests), A/B timing on the workload graphs
M=gpurun_out/s39; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "sddmm or heavy_row or gat_forward or gat_backward" > $M/pytest_sddmm.log 2>&1; echo "pytest rc=$?"; tail -3 $M/pytest_sddmm.log; grep -E "^E " $M/pytest_sddmm.log | head -5
timeout 900 python tools/sddmm_tile_ab.py > $M/ab.log 2>&1; echo "ab rc=$?"; cat $M/ab.log
