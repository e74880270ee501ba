"""ncu per-kernel DRAM traffic -> per-primitive DRAM rate for bench.py's roofline (profiles/ncu_traffic.json).

Input: `ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --cache-control none
--clock-control none --csv` of one bench.py run of a workload.  Every launch of the library's kernels is
attributed to the primitive whose launcher issues it (the tracer's names in bench.py's per_primitive_ms);
the result per primitive is the DRAM bytes moved per millisecond of that primitive's kernel time, which
bench.py multiplies by its own per-call time to report `traffic` (bytes per call).
usage: python tools/ncu_traffic.py <csv> <workload> [profiles/ncu_traffic.json]"""
import csv
import json
import re
import sys

PRIM = [(r"k_spmm", "spmm"), (r"k_sddmm_dot", "sddmm_dot"), (r"k_sddmm|k_seg_|k_heavy_stats|k_row_softmax", "sddmm"),
        (r"k_gat_bwd_a|k_gat_a_combine", "gat_bwd_a"), (r"k_gat_bwd_b|k_gat_b_combine", "gat_bwd_b"),
        (r"k_gat_dz", "gat_dz"), (r"k_gat_der", "gat_der"),
        (r"k_gemm_tn|k_sum_splits", "gemm_tn_tc"), (r"k_gemm_tc|k_prep_b|k_reduce_partials", "gemm_tc")]


def main(path, workload, out="profiles/ncu_traffic.json"):
    rows = [r for r in csv.reader(l for l in open(path) if l.startswith('"'))]
    hdr, rows = rows[0], rows[1:]
    ik, im, iv, iu, iid = (hdr.index(x) for x in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit", "ID"))
    per = {}
    for r in rows:
        k = r[ik]
        if "granii::" not in k:
            continue
        d = per.setdefault(r[iid], {"kernel": k})
        v = float(r[iv].replace(",", ""))
        u = r[iu]
        if r[im] == "gpu__time_duration.sum":
            d["ms"] = v * {"ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "nsecond": 1e-6, "ms": 1.0, "msecond": 1.0}.get(u, 1e-6)
        else:
            d[r[im]] = v * {"byte": 1, "Kbyte": 1e3, "KB": 1e3, "Mbyte": 1e6, "MB": 1e6, "Gbyte": 1e9, "GB": 1e9}.get(u, 1)
    agg = {}
    for d in per.values():
        prim = next((p for pat, p in PRIM if re.search(pat, d["kernel"])), "elementwise")
        a = agg.setdefault(prim, {"ms": 0.0, "bytes": 0.0, "launches": 0})
        a["ms"] += d.get("ms", 0.0)
        a["bytes"] += d.get("dram__bytes_read.sum", 0.0) + d.get("dram__bytes_write.sum", 0.0)
        a["launches"] += 1
    res = {p: {"dram_bytes_per_ms": a["bytes"] / a["ms"], "ncu_kernel_ms": a["ms"], "ncu_dram_bytes": a["bytes"],
               "launches": a["launches"]} for p, a in agg.items() if a["ms"] > 0}
    try:
        tab = json.load(open(out))
    except (OSError, ValueError):
        tab = {}
    tab[workload] = dict(res, _how="ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum "
                         "--cache-control none --clock-control none over one bench.py run (tools/ncu_traffic.py): "
                         "DRAM bytes per ms of each primitive's kernels; bench.py traffic = rate x its own time per call")
    json.dump(tab, open(out, "w"), indent=1)
    print(json.dumps({workload: res}, indent=1))


if __name__ == "__main__":
    main(*sys.argv[1:])
