"""Summarise `ncu --page source --csv --print-source sass` output: top stalled SASS lines."""
import csv
import sys


def main(path, n=25):
    rows = list(csv.reader(open(path)))
    hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
    h = rows[hi]
    data = [r for r in rows[hi + 1:] if r and r[0] != "Address" and len(r) == len(h)]
    si = h.index("Warp Stall Sampling (All Samples)")
    ex = h.index("Instructions Executed")

    def f(x):
        try:
            return float(x)
        except ValueError:
            return 0.0
    tot = sum(f(r[si]) for r in data)
    print("total samples", tot, "instructions", sum(f(r[ex]) for r in data))
    for r in sorted(data, key=lambda r: -f(r[si]))[:n]:
        print(f"{f(r[si]) / tot * 100:5.1f}%  exec={r[ex]:>9}  {r[0]}  {r[1][:120]}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 25)
