"""Write the per-launch DRAM bytes of each kernel of an ncu --set full report into
profiles/ncu_traffic.json under the key "<config>/T<tile>/<path>" (bench.py reads the dominant
kernel's entry for roofline.traffic only when its own config, tile and path match).
python tools/ncu_traffic.py rep.ncu-rep <config> <tile> <path> [source note]"""
import csv
import io
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main(rep, config, tile, path, note=""):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units = rows[0], rows[1]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    per = {}
    for row in rows[2:]:
        d, u = dict(zip(h, row)), dict(zip(h, units))
        name = re.sub(r"^void ", "", d.get("Kernel Name", "?"))
        name = re.sub(r"^zh::", "", name).split("<")[0].split("(")[0]
        b = 0.0
        for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            b += float(d[k].replace(",", "")) * scale.get(u.get(k, "byte"), 1)
        per.setdefault(name, []).append(b)
    p = os.environ.get("ZH_TRAFFIC_JSON", os.path.join(ROOT, "profiles", "ncu_traffic.json"))
    js = json.load(open(p)) if os.path.exists(p) else {}
    if "_source" in js and not isinstance(js["_source"], dict):
        js = {}
    key = f"{config}/T{tile}/{path}"
    js[key] = {k: sum(v) / len(v) for k, v in per.items()}
    js.setdefault("_source", {})[key] = note or f"{os.path.basename(rep)}: dram__bytes_read.sum + dram__bytes_write.sum per launch (mean over captured launches)"
    json.dump(js, open(p, "w"), indent=1, sort_keys=True)
    print(key, js[key])


if __name__ == "__main__":
    main(*sys.argv[1:])
