# segmented row softmax in the entry-tile SDDMM: parity (both paths), A/B
M=gpurun_out/s62; mkdir -p $M
for S in 1 0; do
GRANII_SDDMM_SEG=$S timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "sddmm" > $M/pytest_seg$S.log 2>&1; echo "pytest seg=$S rc=$?"; tail -1 $M/pytest_seg$S.log; grep -E "^E " $M/pytest_seg$S.log | head -5
done
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -q -x -k "sddmm" > $M/pytest_full.log 2>&1; echo "pytest full rc=$?"; tail -1 $M/pytest_full.log; grep -E "^E " $M/pytest_full.log | head -5
timeout 900 python -m pytest tests/test_gpu_multirank.py -q -x -k "gat_forward_backward" > $M/pytest_mr.log 2>&1; echo "pytest mr rc=$?"; tail -1 $M/pytest_mr.log
for S in 0 1; do GRANII_SDDMM_SEG=$S timeout 300 python tools/sddmm_tile_ab.py products,arxiv,pubmed 1 att > $M/ab_seg$S.log 2>&1; echo "seg=$S"; cat $M/ab_seg$S.log; done
