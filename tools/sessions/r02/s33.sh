# dW GEMM accuracy + time vs rows per split
M=gpurun_out/s33; mkdir -p $M
timeout 900 python tools/gemm_tn_err.py 0,512,1024,2048,4096 233000,2449029 > $M/gemm_tn_err.log 2>&1; echo "gemm err rc=$?"; cat $M/gemm_tn_err.log
