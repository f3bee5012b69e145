"""Average DRAM bytes per launch per kernel from an ncu CSV
(--metrics dram__bytes_read.sum,dram__bytes_write.sum,...), merged into
profiles/dram_traffic.json under the given model key.
usage: python scripts/dram_traffic.py <ncu.csv> <model>"""
import csv
import json
import os
import sys
from collections import defaultdict

sys.path.insert(0, os.path.join(os.path.dirname(os.path.abspath(__file__)), ".."))
path, model = sys.argv[1], sys.argv[2]


def solutions_by_node(model):
    """Bound solution name of each node (host-only Algorithm 1 plan): under the
    families packaging a CUfunction serves several solutions, so launches are
    attributed by node order (the capture is exactly one inference)."""
    from paper_conf_dac_huangdxz25_b200 import pask as P
    from paper_conf_dac_huangdxz25_b200.model import DeviceModel
    from workloads import build_model
    spec, _ = build_model(model)
    plan, _ = P.plan(DeviceModel(spec, alloc=False).graph)
    return [P.kernel_name(b[2]) for b in plan]


names = solutions_by_node(model)
per = defaultdict(lambda: defaultdict(float))
ids = []
for r in csv.DictReader(l for l in open(path) if not l.startswith("==")):
    if r.get("Metric Name") in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
        v = float(r["Metric Value"].replace(",", ""))
        unit = r["Metric Unit"]
        v *= {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1024, "MB": 1024 ** 2}.get(unit, 1)
        if r["ID"] not in ids:
            ids.append(r["ID"])
        node = ids.index(r["ID"])
        per[names[node] if node < len(names) else r["Kernel Name"]][r["ID"]] += v
out_path = os.path.join(os.path.dirname(__file__), "..", "profiles", "dram_traffic.json")
data = json.load(open(out_path)) if os.path.exists(out_path) else {}
data["_source"] = ("ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum (default --cache-control all: "
                   "caches flushed before each kernel, the L2-flushed regime of bench.py), one inference, "
                   "bytes per launch averaged over that kernel's launches")
data[model] = {k: int(sum(v.values()) / len(v)) for k, v in per.items()}
json.dump(data, open(out_path, "w"), indent=1)
print(model, data[model])
