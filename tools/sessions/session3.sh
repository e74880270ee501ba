set -u
M=gpurun_out/s3; mkdir -p $M
timeout 900 python tools/gatbwd_sweep.py products > $M/gatbwd_sweep.log 2>&1; echo "gat sweep rc=$?"; cat $M/gatbwd_sweep.log
KS=100,47,256 TUNES="def;4,3;4,4" SLICES="auto" timeout 600 python tools/spmm_sweep.py products > $M/spmm_sweep_products.log 2>&1; echo "spmm sweep rc=$?"; cat $M/spmm_sweep_products.log
