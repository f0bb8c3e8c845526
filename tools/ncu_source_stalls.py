"""Top SASS lines by warp-stall samples in an ncu report (source page): where the warps wait.

  python tools/ncu_source_stalls.py report.ncu-rep [kernel-substring] [top]
"""
import csv
import io
import subprocess
import sys


def main(rep, kern="", top=30):
    txt = subprocess.check_output(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], text=True)
    rows = list(csv.reader(io.StringIO(txt)))
    blocks, cur = [], None
    for r in rows:
        if r and r[0] == "Kernel Name":
            cur = [r[1], None, []]
            blocks.append(cur)
        elif r and r[0] == "Address" and cur is not None:
            cur[1] = r
        elif cur is not None and cur[1] is not None and len(r) == len(cur[1]):
            cur[2].append(r)
    for name, hdr, recs in blocks:
        if kern not in name:
            continue
        si = hdr.index("Warp Stall Sampling (All Samples)")
        tot = sum(float(r[si] or 0) for r in recs)
        print(name[:90], "total samples", tot)
        for i, r in sorted(enumerate(recs), key=lambda x: -float(x[1][si] or 0))[:top]:
            print(f"  {float(r[si] or 0):8.0f} {100 * float(r[si] or 0) / tot:5.1f}%  [{i:5d}] {r[hdr.index('Source')].strip()}")
        break


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else "", int(sys.argv[3]) if len(sys.argv) > 3 else 30)
