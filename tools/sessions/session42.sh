for clb in 1 0 1 0; do GRANII_GATBWD_CLB=$clb CASES="17:100:256" TUNES="def" timeout 900 python tools/gatbwd_sweep.py products 2>&1 | tail -1 | sed "s/^/clb=$clb /"; done
timeout 900 python -m pytest tests -m gpu -x -q -k "gat" 2>&1 | tail -1
