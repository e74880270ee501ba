# dW GEMM accuracy vs reduction length; staged SDDMM softmax parity + timing
M=gpurun_out/s32; mkdir -p $M
timeout 600 python tools/gemm_tn_err.py > $M/gemm_tn_err.log 2>&1; echo "gemm err rc=$?"; cat $M/gemm_tn_err.log
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x -k "sddmm" > $M/pytest_sddmm.log 2>&1; echo "pytest sddmm rc=$?"; tail -3 $M/pytest_sddmm.log
timeout 900 python tools/sddmm_softmax_ab.py 0,100,1024 pubmed,arxiv,products > $M/sddmm_ab.log 2>&1; echo "sddmm ab rc=$?"; cat $M/sddmm_ab.log
