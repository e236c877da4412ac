"""Write profiles/traffic_<tag>.json (read by bench.py) from tools/ncu_metrics.py outputs.
python tools/make_traffic.py TAG NOTE cfg=path/ncu_cfg.json [cfg=...]
traffic = dram__bytes_read.sum + dram__bytes_write.sum of one launch of each kernel."""
import json
import os
import sys

tag, note, pairs = sys.argv[1], sys.argv[2], sys.argv[3:]
out = {"note": note, "traffic_bytes_per_launch": {}}
for p in pairs:
    cfg, path = p.split("=", 1)
    rep = json.load(open(path))
    d = {}
    for k in rep["kernels"]:
        name = k["kernel"].split("::")[-1].split("<")[0].replace("void ", "").replace("_kernel", "")
        if k["dram_read"] is not None:
            d[name] = (k["dram_read"] or 0) + (k["dram_write"] or 0)
    out["traffic_bytes_per_launch"][cfg] = d
root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
dst = os.path.join(root, "profiles", f"traffic_{tag}.json")
json.dump(out, open(dst, "w"), indent=1)
print(dst)
