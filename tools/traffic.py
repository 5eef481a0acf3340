"""Extract per-launch DRAM traffic (dram__bytes_read.sum + write.sum) and
duration from ncu --set full reports into profiles/traffic.json, keyed by
bench config name (the roofline "traffic" field of bench.py).

    python tools/traffic.py C3=gpurun_out/prof_c3.ncu-rep C4=... [--out profiles/traffic.json]
"""
import csv
import io
import json
import subprocess
import sys


def metrics(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))

        def val(name):
            v = float(d[name].replace(",", ""))
            unit = u.get(name, "")
            scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6, "us": 1e-6, "ns": 1e-9, "ms": 1e-3,
                     "msecond": 1e-3}.get(unit, 1)
            return v * scale
        res.append({"kernel": d.get("Kernel Name", "")[:120],
                    "dram_read_bytes": val("dram__bytes_read.sum"),
                    "dram_write_bytes": val("dram__bytes_write.sum"),
                    "duration_s": val("gpu__time_duration.sum")})
    return res


def main():
    outp = "profiles/traffic.json"
    args = [a for a in sys.argv[1:]]
    if "--out" in args:
        i = args.index("--out")
        outp = args[i + 1]
        del args[i:i + 2]
    try:
        data = json.load(open(outp))
    except OSError:
        data = {}
    for a in args:
        name, rep = a.split("=", 1)
        m = metrics(rep)[0]
        data[name] = int(m["dram_read_bytes"] + m["dram_write_bytes"])
        data.setdefault("_detail", {})[name] = m
    json.dump(data, open(outp, "w"), indent=1)
    print(json.dumps(data, indent=1))


if __name__ == "__main__":
    main()
