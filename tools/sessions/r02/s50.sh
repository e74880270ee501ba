# TMA tile::gather4 throughput probe
M=gpurun_out/s50; mkdir -p $M
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/tma_g4 tools/probe/tma_gather4.cu && timeout 120 /tmp/tma_g4 > $M/tma_gather4.jsonl 2>&1; echo "probe rc=$?"; cat $M/tma_gather4.jsonl
