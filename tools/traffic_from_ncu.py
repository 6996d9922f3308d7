"""profiles/traffic.json from an `ncu --set full` capture of the dominant k_search launch (the
bench line's roofline.traffic: DRAM bytes read + written per launch, measured, with its source).
usage: python tools/traffic_from_ncu.py CAPTURE.ncu-rep [out=profiles/traffic.json]"""
import csv
import io
import json
import os
import subprocess
import sys

rep = sys.argv[1]
out = sys.argv[2] if len(sys.argv) > 2 else os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                                       "profiles", "traffic.json")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h, units, v = rows[0], rows[1], rows[2]


def get(name):
    i = h.index(name)
    x = float(v[i].replace(",", ""))
    u = units[i]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
             "msecond": 1e-3, "second": 1.0}.get(u, 1.0)
    return x * scale


rd, wr = get("dram__bytes_read.sum"), get("dram__bytes_write.sum")
t = get("gpu__time_duration.sum")
kname = v[h.index("Kernel Name")]
d = {"k_search_dram_bytes_per_launch": int(rd + wr), "dram_read_bytes": int(rd), "dram_write_bytes": int(wr),
     "launch_seconds": t, "kernel": kname[:120],
     "source": f"ncu --set full capture {os.path.basename(rep)} (query 5478 on C2, tools/profile_one.py)"}
with open(out, "w") as f:
    json.dump(d, f, indent=1)
print(json.dumps(d))
