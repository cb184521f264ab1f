"""Write a roofline-traffic JSON (DRAM bytes per launch) from an ncu report (run here, no GPU needed):
    python tools/traffic_from_ncu.py rep.ncu-rep out.json "kernel description" algorithmic_bytes"""
import csv
import io
import json
import subprocess
import sys

rep, out, desc, alg = sys.argv[1], sys.argv[2], sys.argv[3], int(sys.argv[4])
txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics",
                      "dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,Kernel Name"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(txt)))
hdr, units, vals = rows[0], rows[1], rows[2]


def get(name):
    i = hdr.index(name)
    v = float(vals[i].replace(",", ""))
    u = units[i]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6, "usecond": 1e-6,
             "msecond": 1e-3, "ms": 1e-3, "nsecond": 1e-9, "second": 1.0}.get(u, 1)
    return v * scale


r, w, t = get("dram__bytes_read.sum"), get("dram__bytes_write.sum"), get("gpu__time_duration.sum")
json.dump({"kernel": desc, "dram_bytes_per_launch": r + w, "parts": {"read": r, "write": w},
           "duration_s": t, "algorithmic_bytes": alg, "traffic_over_algorithmic": (r + w) / alg,
           "source": rep}, open(out, "w"), indent=1)
print(open(out).read())
