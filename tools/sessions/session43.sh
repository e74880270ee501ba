for cl in 1 0 1 0; do GRANII_GATBWD_CL=$cl CASES="16:64:256;16:64:512" TUNES="def" timeout 900 python tools/gatbwd_sweep.py products 2>&1 | tail -2 | sed "s/^/cl=$cl /"; done
timeout 900 python -m pytest tests -m gpu -x -q -k "gat" 2>&1 | tail -1
