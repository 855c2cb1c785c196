"""Extract the roofline traffic of one profiled worker launch from an .ncu-rep
into profiles/ncu_worker_traffic.json (read by bench.py for roofline.traffic)."""
import csv
import io
import json
import subprocess
import sys

rep, workload, out = sys.argv[1], sys.argv[2], sys.argv[3]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h, units, vals = rows[0], rows[1], rows[2]


def get(name, scale=1.0):
    i = h.index(name)
    v = float(vals[i].replace(",", ""))
    u = units[i]
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "nsecond": 1e-9,
            "usecond": 1e-6, "msecond": 1e-3, "second": 1.0, "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1.0}.get(u, 1.0)
    return v * mult * scale


rd = get("dram__bytes_read.sum")
wr = get("dram__bytes_write.sum")
dur = get("gpu__time_duration.sum")
res = {"workload": workload, "kernel": h and vals[h.index("Kernel Name")],
       "dram_bytes_read": rd, "dram_bytes_write": wr, "dram_bytes_per_launch": rd + wr,
       "ncu_duration_s": dur, "source": rep.split("/")[-1],
       "note": "one ncu --set full capture (application replay, --profile-from-start off) of the worker launch"}
json.dump(res, open(out, "w"), indent=1)
print(json.dumps(res))
