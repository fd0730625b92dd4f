"""Summarise an ncu --metrics gpu__time_duration.sum --csv launch list: share of GPU time per kernel."""
import collections
import csv
import sys


def main(path, out=None, top=40):
    rows = list(csv.reader(open(path)))
    hi = [i for i, r in enumerate(rows) if r and r[0] == "ID"][0]
    h = rows[hi]
    ki, mi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    scale = {"ns": 1e-6, "nsecond": 1e-6, "us": 1e-3, "usecond": 1e-3, "ms": 1.0, "msecond": 1.0}
    tot, cnt = collections.defaultdict(float), collections.Counter()
    for r in rows[hi + 1:]:
        if len(r) <= mi:
            continue
        v = float(r[mi].replace(",", "")) * scale.get(r[ui], 1e-6)
        tot[r[ki][:110]] += v
        cnt[r[ki][:110]] += 1
    T = sum(tot.values())
    lines = [f"total {T:.2f} ms over {sum(cnt.values())} launches"]
    for k, v in sorted(tot.items(), key=lambda x: -x[1])[:top]:
        lines.append(f"{v / T * 100:6.2f}% {v:9.3f} ms n={cnt[k]:5d} {k}")
    text = "\n".join(lines)
    if out:
        with open(out, "w") as f:
            w = csv.writer(f)
            w.writerow(["share_pct", "total_ms", "launches", "kernel"])
            for k, v in sorted(tot.items(), key=lambda x: -x[1]):
                w.writerow([f"{v / T * 100:.3f}", f"{v:.3f}", cnt[k], k])
    print(text)


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else None)
