# GAT backward on graphs with empty rows (no self-loops, isolated nodes)
M=gpurun_out/s60; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py -q -k "empty_rows" > $M/pytest.log 2>&1; echo "pytest rc=$?"; tail -3 $M/pytest.log; grep -E "^E |Error|assert" $M/pytest.log | head -10
