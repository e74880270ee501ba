# final check of HEAD: smoke + the whole GPU suite
M=gpurun_out/s64; mkdir -p $M
python -c "import __graft_entry__ as g; g.smoke()" > $M/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 $M/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > $M/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $M/pytest_gpu.log; grep -E "^E " $M/pytest_gpu.log | head -5
