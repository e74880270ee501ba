"""Copy one round_measure.sh session (gpurun_out/<M>) into profiles/r01 and print the status table
rows of DESIGN.md §10 (ms/step, G edges/s, selected compositions, max regret)."""
import glob
import json
import os
import shutil
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
src = os.path.join(ROOT, "gpurun_out", sys.argv[1] if len(sys.argv) > 1 else "m3")
dst = os.path.join(ROOT, "profiles", "r01")
for f in glob.glob(os.path.join(src, "bench_*.json")) + glob.glob(os.path.join(src, "scaling_projection_*.json")):
    shutil.copy(f, dst)
for f, g in (("regret_sweep.json", "regret_sweep.json"), ("ncu_launches_default_bench.txt", None),
             ("ncu_launches_share.json", None), ("spmm_full_summary.json", "ncu_spmm_full_summary.json"),
             ("gemm_full_summary.json", "ncu_gemm_full_summary.json"),
             ("gat_train_full_summary.json", "ncu_products_gat_train_summary.json"),
             ("calib.log", "calibration_report.txt")):
    p = os.path.join(src, f)
    if os.path.exists(p):
        shutil.copy(p, os.path.join(dst, g or f))
for f in ("b200.txt", "b200_samples.json"):
    p = os.path.join(src, f)
    if os.path.exists(p):
        shutil.copy(p, os.path.join(ROOT, "calib", f))
for f in sorted(glob.glob(os.path.join(src, "bench_*.json"))):
    d = json.load(open(f))
    sel = d.get("selector", {})
    reg = max([v.get("regret", 0.0) for v in sel.values()] or [0.0])
    print(f"| {d['config']['workload']} | {d['ms_per_step']:.3f} | {d['value'] / 1e9:.2f} | "
          f"{', '.join(c.replace('GCN_', '').replace('GAT_', '') for c in d['config'].get('compositions', []))} | "
          f"{100 * reg:.1f} % | {d['roofline']['kernel']} {d['roofline']['frac']:.2f} |")
r = os.path.join(src, "regret_sweep.json")
if os.path.exists(r):
    print(json.dumps(json.load(open(r)).get("summary"), indent=1))
