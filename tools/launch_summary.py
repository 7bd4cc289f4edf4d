"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv): per kernel count,
total and mean device time and share of the listed time."""
import collections
import csv
import sys


def summary(path):
    rows = [r for r in csv.reader(open(path)) if len(r) > 5]
    h = rows[0]
    ki, mi, vi = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value")
    tot = collections.defaultdict(float)
    cnt = collections.Counter()
    for r in rows[1:]:
        if r[mi] == "gpu__time_duration.sum":
            k = r[ki].split("(")[0].replace("scanb200::", "").replace("<unnamed>::", "")
            tot[k] += float(r[vi].replace(",", ""))
            cnt[k] += 1
    s = sum(tot.values())
    out = ["%s: %d launches, %.1f us listed" % (path, sum(cnt.values()), s / 1e3)]
    for k in sorted(tot, key=lambda k: -tot[k]):
        out.append("  %-58s n=%4d  mean=%9.2f us  share=%5.1f%%" % (k[:58], cnt[k], tot[k] / cnt[k] / 1e3, 100 * tot[k] / s))
    return "\n".join(out)


if __name__ == "__main__":
    for p in sys.argv[1:]:
        print(summary(p))
