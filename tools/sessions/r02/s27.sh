M=gpurun_out/s27; mkdir -p $M
timeout 2400 python -m pytest tests -m gpu -x -q --durations=15 > $M/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -22 $M/pytest_gpu.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > $M/smoke.log 2>&1; echo "smoke rc=$?"; tail -2 $M/smoke.log
