set -u
M=gpurun_out/s4; mkdir -p $M
CASES="16:100:256;16:64:512;17:100:256;16:256:47" TUNES="def;8,4,2;16,2,2;16,4,2;16,4,1;32,2,2;32,2,1;32,4,2;32,4,1;16,8,1" timeout 1200 python tools/gatbwd_sweep.py products > $M/gatbwd_sweep.log 2>&1; echo "gat sweep rc=$?"; cat $M/gatbwd_sweep.log
CASES="16:64:256;17:64:256;16:128:512" TUNES="def;8,4,2;16,2,2;16,4,2;16,4,1;32,2,2;32,2,1;32,4,2;32,4,1" timeout 600 python tools/gatbwd_sweep.py arxiv > $M/gatbwd_sweep_arxiv.log 2>&1; echo "gat sweep arxiv rc=$?"; cat $M/gatbwd_sweep_arxiv.log
