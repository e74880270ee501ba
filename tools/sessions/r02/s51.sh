# GAT backward: deeper per-group unroll (U = 4) now that the 32-bit masks freed registers
M=gpurun_out/s51; mkdir -p $M
CASES="16:256:47:1" TUNES="def;8,2,4,0;8,2,4,4;8,2,4,3;8,2,2,0;def" timeout 900 python tools/gatbwd_sweep.py products > $M/sweep_k47.log 2>&1; echo "sweep47 rc=$?"; cat $M/sweep_k47.log
CASES="17:100:256:0" TUNES="def;16,2,4,0,1;16,2,4,4,1;16,2,2,4,1;def" timeout 900 python tools/gatbwd_sweep.py products > $M/sweep_k100.log 2>&1; echo "sweep100 rc=$?"; cat $M/sweep_k100.log
