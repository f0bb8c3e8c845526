"""Write profiles/<name>.json with the DRAM bytes per launch of the FI replica kernels from ncu
--set full reports (one launch each): {kernel: {dram_bytes_per_launch, replicas_per_launch, source}}.

  python tools/traffic_json.py out.json tpacf=report1.ncu-rep:64 mriq=report2.ncu-rep:76
"""
import csv
import io
import json
import subprocess
import sys


def dram(rep):
    txt = subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv"], text=True)
    rows = list(csv.reader(io.StringIO(txt)))
    h, u, v = rows[0], rows[1], rows[2]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    tot = 0.0
    for k in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
        j = h.index(k)
        tot += float(v[j].replace(",", "")) * scale[u[j]]
    return tot, v[h.index("Kernel Name")]


def main(out, *specs):
    res = {}
    for sp in specs:
        name, rest = sp.split("=", 1)
        rep, reps = rest.rsplit(":", 1)
        b, kern = dram(rep)
        res[f"{name}_fi_kernel"] = {"dram_bytes_per_launch": int(b), "replicas_per_launch": int(reps),
                                    "source": f"ncu --set full --clock-control none, tools/profile_fi.py {name} ({rep}): "
                                              f"dram__bytes_read.sum + dram__bytes_write.sum of one launch of {kern[:60]}"}
    with open(out, "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main(*sys.argv[1:])
