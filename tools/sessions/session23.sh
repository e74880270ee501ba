set -u
M=gpurun_out/${SESS:-s23}; mkdir -p $M
timeout 1200 python -m pytest tests -m gpu -x -q -k "gat" > $M/pytest.log 2>&1; echo "pytest rc=$?"; tail -2 $M/pytest.log
CASES="17:100:256;16:256:47;16:100:256" TUNES="def" timeout 900 python tools/gatbwd_sweep.py products 2>&1 | tail -3
CASES="16:64:256;17:64:256" TUNES="def" timeout 900 python tools/gatbwd_sweep.py pubmed 2>&1 | tail -2
