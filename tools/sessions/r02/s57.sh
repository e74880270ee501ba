# source-level ncu of the entry-tile SDDMM (scores + softmax) on products
M=gpurun_out/s57; mkdir -p $M
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"k_sddmm1_tile" -s 1 -c 1 -o /tmp/st python tools/sddmm_tile_ab.py products 1 att > $M/st.log 2>&1; echo "ncu rc=$?"
ncu -i /tmp/st.ncu-rep --page source --csv --print-source sass > $M/st_sass.csv 2>/dev/null
ncu -i /tmp/st.ncu-rep --page raw --csv > $M/st_raw.csv 2>/dev/null
python tools/ncu_summary.py /tmp/st.ncu-rep > $M/st_summary.json; cat $M/st_summary.json | grep -E "time_ms|issue|warps_active|l1_pct|l2_pct|dram_pct"
