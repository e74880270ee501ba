M=gpurun_out/s29; mkdir -p $M
timeout 600 python tools/csr_time.py > $M/csr_time.log 2>&1; echo "csr rc=$?"; cat $M/csr_time.log
timeout 900 python tools/gat_grad_err.py > $M/gat_grad_err.log 2>&1; echo "err rc=$?"; cat $M/gat_grad_err.log | tail -20
