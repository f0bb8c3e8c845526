"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv --log-file X) per kernel:
launches, total device time and share.  ncu serialises and cold-starts every launch, so only the
SHARES are comparable with bench.py's live numbers."""
import collections
import csv
import re
import sys


def main(path, header=""):
    rows = list(csv.reader(open(path)))
    i = next(k for k, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[i]
    kn, mn, mv, mu = (hdr.index(c) for c in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit"))
    tot = collections.Counter()
    cnt = collections.Counter()
    for r in rows[i + 1:]:
        if len(r) <= mv or r[mn] != "gpu__time_duration.sum":
            continue
        name = re.sub(r"<.*>", "<..>", r[kn].split("(")[0])
        v = float(r[mv].replace(",", ""))
        v *= {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}.get(r[mu], 1.0)
        tot[name] += v
        cnt[name] += 1
    s = sum(tot.values())
    out = [header] if header else []
    out.append(f"# {sum(cnt.values())} launches; cold-cache, serialised -> compare SHARES")
    for name, v in tot.most_common():
        out.append(f"{name:45s} launches={cnt[name]:5d} total_us={v:11.1f} share={100 * v / s:5.1f}%")
    print("\n".join(out))


if __name__ == "__main__":
    main(sys.argv[1], " ".join(sys.argv[2:]))
