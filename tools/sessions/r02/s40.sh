# random 4-byte gather rate probe (the K=1 SDDMM roof); ncu of both K=1 SDDMM kernels on products
M=gpurun_out/s40; mkdir -p $M
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/gather_rate tools/probe/gather_rate.cu && timeout 300 /tmp/gather_rate > $M/gather_rate.json; echo "probe rc=$?"; cat $M/gather_rate.json
for T in 0 1; do
timeout 600 ncu --set full --clock-control none -k regex:"k_sddmm1" -s 2 -c 2 -o /tmp/sd$T python tools/sddmm_tile_ab.py products $T att > /dev/null 2>&1; echo "ncu $T rc=$?"
python tools/ncu_summary.py /tmp/sd$T.ncu-rep > $M/ncu_sddmm_tile$T.json
ncu -i /tmp/sd$T.ncu-rep --page raw --csv > $M/ncu_sddmm_tile${T}_raw.csv 2>/dev/null
done
