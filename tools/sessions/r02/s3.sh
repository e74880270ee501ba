M=gpurun_out/s3; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "directed or transpose" > $M/pytest_dir.log 2>&1; echo "dir rc=$?"; tail -5 $M/pytest_dir.log
timeout 900 python -m pytest tests/test_gpu_multirank.py -x -q -k "directed or watchdog or query" > $M/pytest_mr.log 2>&1; echo "mr rc=$?"; tail -5 $M/pytest_mr.log
