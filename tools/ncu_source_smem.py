"""Per-instruction shared-memory wavefronts from an ncu report (source page, SASS): the hot
shared-memory instructions with executed count, wavefronts, ideal wavefronts and N-way conflicts.

  python tools/ncu_source_smem.py report.ncu-rep [top]
"""
import csv
import io
import subprocess
import sys


def main(rep, top=25):
    txt = subprocess.check_output(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], text=True)
    rows = list(csv.reader(io.StringIO(txt)))
    k = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
    hdr = rows[k]
    col = {n: hdr.index(n) for n in hdr}
    recs = []
    for r in rows[k + 1:]:
        if len(r) < len(hdr):
            continue
        try:
            wf = float(r[col["L1 Wavefronts Shared"]] or 0)
        except ValueError:
            continue
        if wf <= 0:
            continue
        ex = float(r[col["Instructions Executed"]] or 0)
        ideal = float(r[col["L1 Wavefronts Shared Ideal"]] or 0)
        recs.append((wf, ex, ideal, r[col["Source"]].strip()))
    tot = sum(x[0] for x in recs)
    print(f"total shared wavefronts {tot:.4g}")
    by = {}
    for wf, ex, ideal, src in recs:
        op = src.split()[0] if not src.startswith("@") else src.split()[1]
        a = by.setdefault(op, [0.0, 0.0, 0.0])
        a[0] += wf; a[1] += ex; a[2] += ideal
    for op, (wf, ex, ideal) in sorted(by.items(), key=lambda kv: -kv[1][0]):
        print(f"  {op:22s} wavefronts {wf:12.4g} ({100 * wf / tot:5.1f} %)  executed {ex:12.4g}  per instr {wf / max(ex, 1):5.2f}  ideal/instr {ideal / max(ex, 1):5.2f}")
    for wf, ex, ideal, src in sorted(recs, reverse=True)[:top]:
        print(f"  {wf:12.4g} {ex:12.4g} {wf / max(ex, 1):5.2f} {ideal / max(ex, 1):5.2f}  {src}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 25)
