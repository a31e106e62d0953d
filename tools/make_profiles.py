"""Turn gpurun_out ncu captures into committed summaries under profiles/:
   profiles/<tag>_ncu_summary.json  (per capture: key metrics + stall mix)
   profiles/ncu_traffic.json        (workload/engine -> dram read+write bytes per launch, for bench.py)
   profiles/<tag>_launches_summary.json (share of each kernel in the bench launch list)"""
import csv, glob, json, os, re, sys
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_summary import summarise

tag = sys.argv[1]
root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
out = {}
traffic_path = os.path.join(root, "profiles", "ncu_traffic.json")
traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
def mbytes(s):
    v, u = s.split()[0], s.split()[1] if len(s.split()) > 1 else "byte"
    f = float(v)
    return f * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
for rep in sorted(glob.glob(os.path.join(root, "gpurun_out", f"{tag}_*.ncu-rep"))):
    name = os.path.basename(rep)[len(tag) + 1:-len(".ncu-rep")]
    s = summarise(rep)
    out[name] = s
    m = re.match(r"(.+)_(tc|rdg_cuda|direct|auto)(_k\d+)?$", name)
    if m and s:
        d = s[0]
        traffic[f"{m.group(1)}/{m.group(2)}"] = {
            "bytes": mbytes(d["dram__bytes_read.sum"]) + mbytes(d["dram__bytes_write.sum"]),
            "kernel": d["kernel"], "source": f"profiles/{tag}_ncu_summary.json", "fuse": (m.group(3) or "_k1")[2:]}
json.dump(out, open(os.path.join(root, "profiles", f"{tag}_ncu_summary.json"), "w"), indent=1)
json.dump(traffic, open(traffic_path, "w"), indent=1)
lp = os.path.join(root, "gpurun_out", f"{tag}_launches.csv")
if os.path.exists(lp):
    rows = [r for r in csv.reader(open(lp)) if len(r) > 5]
    hdr = rows[0]
    ki, vi, ni = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Name")
    agg = {}
    for r in rows[1:]:
        if r[ni] != "gpu__time_duration.sum":
            continue
        k = r[ki].split("(")[0][:80]
        a = agg.setdefault(k, [0, 0.0])
        a[0] += 1; a[1] += float(r[vi].replace(",", ""))
    tot = sum(v[1] for v in agg.values())
    summ = {k: {"launches": v[0], "time": v[1], "share": v[1] / tot} for k, v in sorted(agg.items(), key=lambda x: -x[1][1])}
    json.dump({"unit": "ns (ncu gpu__time_duration.sum, cold-cache serialised)", "kernels": summ},
              open(os.path.join(root, "profiles", f"{tag}_launches_summary.json"), "w"), indent=1)
print("ok", list(out))
