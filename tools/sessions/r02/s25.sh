M=gpurun_out/s25; mkdir -p $M
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --no-cold"
for sl in 32 64 128; do GRANII_SPMM_SLICE=$sl timeout 600 $B --out $M/reddit_sl$sl.json > /dev/null 2>&1; done
for sl in 32 64; do GRANII_SPMM_SLICE=$sl timeout 600 $B --workload reddit-gcn2-train-h1024 --out $M/h1024_sl$sl.json > /dev/null 2>&1; done
python tools/ab_summary.py $M/*.json
