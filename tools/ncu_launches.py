"""ncu launch list (--metrics gpu__time_duration.sum --csv) -> profiles text list + per-kernel share JSON.
usage: python tools/ncu_launches.py launches.csv out.txt out_share.json "<command that was profiled>" """
import csv
import json
import re
import sys

src, out_txt, out_json, cmd = sys.argv[1:5]
rows = [r for r in csv.reader(l for l in open(src) if l.startswith('"'))]
hdr, rows = rows[0], rows[1:]
ik, iv, iu = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")


def short(n):
    n = re.sub(r"\(.*\)$", "", n) if n.startswith("void ") else n
    return n.replace("void ", "").replace("at::", "").strip()


launches = []
for r in rows:
    us = float(r[iv].replace(",", "")) / (1000.0 if r[iu] == "ns" else (1e-3 if r[iu] == "ms" else 1.0))
    launches.append((short(r[ik]), us))
with open(out_txt, "w") as f:
    f.write(f"# ncu --metrics gpu__time_duration.sum --clock-control none of\n#   {cmd}\n")
    f.write("# (whole process incl. setup; per-launch times are cold-cache and serialised: compare SHARES)\n")
    f.write("# launch_index kernel duration_us\n")
    for i, (k, us) in enumerate(launches):
        f.write(f"{i} {k} {us:.2f}\n")
agg = {}
for k, us in launches:
    if "granii::" not in k:
        continue
    a = agg.setdefault(k, {"launches": 0, "us": 0.0})
    a["launches"] += 1
    a["us"] += us
tot = sum(a["us"] for a in agg.values())
for a in agg.values():
    a["us"] = round(a["us"], 1)
    a["share_of_granii_time"] = round(a["us"] / tot, 4)
json.dump(dict(sorted(agg.items(), key=lambda kv: -kv[1]["us"])), open(out_json, "w"), indent=1)
print(json.dumps(dict(list(sorted(agg.items(), key=lambda kv: -kv[1]["us"]))[:6]), indent=1))
