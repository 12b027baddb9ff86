"""Summarise an `ncu --metrics gpu__time_duration.sum --csv` launch list per kernel (shares of the step)."""
import collections
import csv
import sys

SCALE = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0, "s": 1e3, "second": 1e3}


def main(path, header=""):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if "Kernel Name" in r][0]
    hdr = rows[hi]
    ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    tot, cnt = collections.defaultdict(float), collections.Counter()
    for r in rows[hi + 1:]:
        if len(r) <= vi:
            continue
        name = r[ki].split("(")[0].replace("void ", "")
        tot[name] += float(r[vi].replace(",", "")) * SCALE.get(r[ui], 1.0)
        cnt[name] += 1
    T = sum(tot.values())
    out = [header] if header else []
    out.append(f"{'kernel':45s} {'launches':>8s} {'total_ms':>10s} {'share%':>7s} {'avg_ms':>9s}")
    for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
        out.append(f"{k:45s} {cnt[k]:8d} {v:10.3f} {100 * v / T:7.1f} {v / cnt[k]:9.3f}")
    out.append(f"total {T:.3f} ms over {sum(cnt.values())} launches")
    print("\n".join(out))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else "")
