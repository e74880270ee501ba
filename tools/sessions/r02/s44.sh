# random-row gather DRAM roof; per-primitive prediction breakdown of the selector's misses; the GPU suite on the
# reverted kernels; regret sweep with the Horner addend feature
M=gpurun_out/s44; mkdir -p $M
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/gather_rate tools/probe/gather_rate.cu && timeout 300 /tmp/gather_rate > $M/gather_rate.json; echo "probe rc=$?"; cat $M/gather_rate.json
timeout 600 python tools/prim_breakdown.py belgium tagcn 256 256 arxiv gat 256 512 > $M/prim_breakdown.jsonl 2> $M/prim_breakdown.err; echo "breakdown rc=$?"; cat $M/prim_breakdown.jsonl | cut -c1-900
timeout 1500 python -m pytest tests -m gpu -x -q > $M/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 $M/pytest_gpu.log; grep -E "^E " $M/pytest_gpu.log | head -5
timeout 1800 python tools/regret_sweep.py $M/regret_sweep.json > $M/regret_sweep.log 2>&1; echo "regret sweep rc=$?"; tail -4 $M/regret_sweep.log
