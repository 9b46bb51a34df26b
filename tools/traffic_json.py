#!/usr/bin/env python
"""Write profiles/traffic.json (DRAM bytes per launch, from ncu --set full captures) that bench.py
reports as roofline.traffic.

usage: python tools/traffic_json.py "<source note>" gpurun_out/prof_*.ncu-rep > profiles/traffic.json
"""
import csv
import io
import json
import subprocess
import sys


def main():
    note, reps = sys.argv[1], sys.argv[2:]
    out = {}
    for rep in reps:
        txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
        rows = list(csv.reader(io.StringIO(txt)))
        hdr = rows[0]
        for r in rows[2:]:
            name = r[hdr.index("Kernel Name")].split("(")[0]
            for pre in ("void ", "gpa::", "<unnamed>::", "unnamed>::", "(anonymous namespace)::"):
                name = name.replace(pre, "")
            f = lambda m: float(r[hdr.index(m)].replace(",", ""))
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
            u = rows[1]
            rd = f("dram__bytes_read.sum") * scale.get(u[hdr.index("dram__bytes_read.sum")], 1)
            wr = f("dram__bytes_write.sum") * scale.get(u[hdr.index("dram__bytes_write.sum")], 1)
            t = f("gpu__time_duration.sum")
            tu = u[hdr.index("gpu__time_duration.sum")]
            ms = t / 1e6 if tu == "ns" else t / 1e3 if tu == "us" else t if tu == "ms" else t * 1e3
            out.setdefault(name, {"dram_bytes": rd + wr, "ncu_ms": ms})
    out["_source"] = note
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
