M=gpurun_out/s15; mkdir -p $M
cd tools && timeout 900 python prim_breakdown.py arxiv gat 256 512 arxiv gat 64 512 reddit tagcn 602 256 reddit gcn 602 256 belgium tagcn 256 256 belgium sgc 256 256 > ../$M/breakdown.jsonl 2> ../$M/breakdown.err; echo "rc=$?"; tail -3 ../$M/breakdown.err
