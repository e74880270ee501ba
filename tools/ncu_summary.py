"""Summarise an ncu report (raw page) into a compact table: one row per profiled kernel."""
import csv, io, json, subprocess, sys
KEYS = {
    "time_ms": ("gpu__time_duration.sum", 1e-6),
    "dram_read_MB": ("dram__bytes_read.sum", 1e-6),
    "dram_write_MB": ("dram__bytes_write.sum", 1e-6),
    "dram_pct": ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", 1),
    "l2_hit_pct": ("lts__t_sector_hit_rate.pct", 1),
    "l2_pct": ("lts__throughput.avg.pct_of_peak_sustained_elapsed", 1),
    "l1_pct": ("l1tex__throughput.avg.pct_of_peak_sustained_active", 1),
    "sm_pct": ("sm__throughput.avg.pct_of_peak_sustained_elapsed", 1),
    "issue_pct": ("smsp__issue_active.avg.pct_of_peak_sustained_active", 1),
    "warps_active_pct": ("sm__warps_active.avg.pct_of_peak_sustained_active", 1),
    "regs": ("launch__registers_per_thread", 1),
    "inst_M": ("smsp__inst_executed.sum", 1e-6),
    "l2_sectors_M": ("lts__t_sectors.sum", 1e-6),
    "tensor_pct": ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", 1),
    "stall_long_sb": ("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio", 1),
}
def unit_scale(u):
    return {"usecond": 1e3, "us": 1e3, "msecond": 1e6, "ms": 1e6, "nsecond": 1, "ns": 1, "second": 1e9, "s": 1e9,
            "Kbyte": 1e3, "KB": 1e3, "Mbyte": 1e6, "MB": 1e6, "Gbyte": 1e9, "GB": 1e9, "byte": 1}.get(u, 1)
def main(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")][:60]}
        for k, (m, sc) in KEYS.items():
            if m in hdr:
                i = hdr.index(m)
                try:
                    v = float(r[i].replace(",", ""))
                except ValueError:
                    continue
                if k.endswith("_ms"):
                    v = v * unit_scale(units[i]) * 1e-6
                elif k.endswith("_MB"):
                    v = v * unit_scale(units[i]) * 1e-6
                else:
                    v = v * sc
                d[k] = round(v, 4)
        res.append(d)
    return res
if __name__ == "__main__":
    res = main(sys.argv[1])
    print(json.dumps(res, indent=1))
