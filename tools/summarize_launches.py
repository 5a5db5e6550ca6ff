"""ncu launch list (--metrics gpu__time_duration.sum --csv) -> markdown table of
per-kernel launches, mean/total ns and share of the listed time."""
import collections
import csv
import sys


def main(path, out, title=None):
    rows = []
    with open(path) as f:
        lines = [ln for ln in f if ln.startswith('"')]
    for r in csv.DictReader(lines):
        if r.get("Metric Name") == "gpu__time_duration.sum":
            rows.append((r["Kernel Name"], float(r["Metric Value"].replace(",", ""))))
    agg = collections.OrderedDict()
    for k, v in rows:
        a = agg.setdefault(k, [0, 0.0])
        a[0] += 1
        a[1] += v
    total = sum(v for _, v in rows) or 1.0
    with open(out, "w") as f:
        f.write(f"# ncu launch list (gpu__time_duration.sum, --clock-control none): `{title or path}`\n\n")
        f.write("Cold-cache, serialized launches: compare SHARES, not absolute times.\n\n")
        f.write("| kernel | launches | mean ns | total ns | share |\n|---|---|---|---|---|\n")
        for k, (c, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
            f.write(f"| `{k[:90]}` | {c} | {t / c:.1f} | {t:.1f} | {t / total:.3f} |\n")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], sys.argv[3] if len(sys.argv) > 3 else None)
