"""Summarise an `ncu --page source --csv` export: stall-reason totals and the top SASS lines."""
import csv
import sys


def main(path, top=25):
    rows = list(csv.reader(open(path)))
    h = rows[1]
    ks = h.index("Warp Stall Sampling (All Samples)")
    cols = [k for k, x in enumerate(h) if x.startswith("stall_") and "Not Issued" not in x]
    data = []
    for r in rows[2:]:
        try:
            data.append((float(r[ks] or 0), r))
        except (ValueError, IndexError):
            pass
    tot = sum(v for v, _ in data) or 1.0
    agg = {}
    for _, r in data:
        for k in cols:
            agg[h[k]] = agg.get(h[k], 0.0) + float(r[k] or 0)
    print("stalls:", ", ".join(f"{k[6:]} {100 * v / tot:.1f}%" for k, v in sorted(agg.items(), key=lambda t: -t[1])[:8]))
    data.sort(key=lambda t: -t[0])
    for v, r in data[:top]:
        top_k = max(cols, key=lambda k: float(r[k] or 0))
        print(f"{100 * v / tot:5.1f}% {r[0][-5:]} {r[1].strip()[:70]:70s} {h[top_k][6:]}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 25)
