M=gpurun_out/s7; mkdir -p $M
B="python bench.py --steps 10 --warmup 3 --no-e2e --no-cpu --no-regret --no-cold"
for v in "o1" "n1m5" "n1m6" "n1m8" "n2m4" "n2m6"; do
  case $v in o1) E="GRANII_SDDMM_ORDERED=1";; n1m5) E="GRANII_SDDMM_NR=1 GRANII_SDDMM_MINB=5";; n1m6) E="GRANII_SDDMM_NR=1 GRANII_SDDMM_MINB=6";;
    n1m8) E="GRANII_SDDMM_NR=1 GRANII_SDDMM_MINB=8";; n2m4) E="GRANII_SDDMM_NR=2 GRANII_SDDMM_MINB=4";; n2m6) E="GRANII_SDDMM_NR=2 GRANII_SDDMM_MINB=6";; esac
  env $E GRANII_GAT_FUSED=0 timeout 600 $B --workload products-gat2-infer --out $M/gatunf_$v.json > $M/gatunf_$v.log 2>&1
  env $E timeout 600 $B --workload arxiv-gat-infer --out $M/arxiv_$v.json > $M/arxiv_$v.log 2>&1
done
python tools/ab_summary.py $M/*.json
