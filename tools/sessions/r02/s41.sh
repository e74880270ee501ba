# tile SDDMM with register-resident short rows: parity + LPG sweep
M=gpurun_out/s41; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "sddmm or heavy_row" > $M/pytest_sddmm.log 2>&1; echo "pytest rc=$?"; tail -2 $M/pytest_sddmm.log; grep -E "^E " $M/pytest_sddmm.log | head -5
timeout 300 python tools/sddmm_tile_ab.py pubmed,arxiv,reddit,products 0 > $M/ab_old.log 2>&1; cat $M/ab_old.log
for L in 4 8 16 32; do GRANII_SDDMM_TILE_LPG=$L timeout 300 python tools/sddmm_tile_ab.py pubmed,arxiv,reddit,products 1 > $M/ab_lpg$L.log 2>&1; echo "LPG $L"; cat $M/ab_lpg$L.log; done
