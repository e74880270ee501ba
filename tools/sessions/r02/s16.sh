M=gpurun_out/s16; mkdir -p $M
timeout 900 python -m pytest tests/test_gpu_multirank.py -x -q -k "phase or partitioned" > $M/pytest_mr.log 2>&1; echo "mr rc=$?"; tail -2 $M/pytest_mr.log
for wl in products-gcn2-infer reddit-gcn2-train products-gat2-infer; do
  timeout 900 python tools/scaling_projection.py --workload $wl --gpus 1,2,4,8 --ranks 0,7 --bw_gbs 725 --out $M/proj_$wl.json > $M/proj_$wl.log 2>&1; echo "proj $wl rc=$?"
  python -c "
import json; d=json.load(open('$M/proj_$wl.json'))
for G,v in d['per_G'].items(): print('$wl', G, 'compute %.3f comm %.3f no_ovl %.3f ovl_bound %.3f' % (v['max_rank_compute_ms'], v['modelled_comm_ms'], v['no_overlap_ms'], v['overlap_bound_ms']), v['ranks'][0].get('plan', {}))
"
done
