"""Top SASS instructions of an ncu source-page CSV (tools/ab_ncu.sh) by samples, wavefronts, conflicts.

  python tools/ncu_src_top.py gpurun_out/ab_new1_src.csv [N]
"""
import csv
import sys


def main():
    path = sys.argv[1]
    N = int(sys.argv[2]) if len(sys.argv) > 2 else 25
    lines = open(path).read().split("\n")
    start = [i for i, l in enumerate(lines) if l.startswith('"Address"')][0]
    rows = list(csv.reader(lines[start:]))
    hdr = rows[0]
    ix = {k: i for i, k in enumerate(hdr)}
    data = [r for r in rows[1:] if len(r) == len(hdr)]

    def f(r, k):
        try:
            return float(r[ix[k]])
        except (KeyError, ValueError):
            return 0.0
    tot = sum(f(r, "# Samples") for r in data)
    print(f"samples {tot:.0f}, instructions {sum(f(r, 'Instructions Executed') for r in data):.3e}")
    cols = ["# Samples", "Instructions Executed", "L1 Wavefronts Shared", "L1 Wavefronts Shared Excessive",
            "L1 Tag Requests Global", "stall_long_sb", "stall_short_sb", "stall_mio", "stall_wait"]
    for title, key in (("samples", "# Samples"), ("shared excessive", "L1 Wavefronts Shared Excessive"),
                       ("global tag requests", "L1 Tag Requests Global")):
        print(f"== top by {title}")
        for r in sorted(data, key=lambda r: -f(r, key))[:N if key == "# Samples" else 12]:
            if f(r, key) <= 0:
                break
            print("  " + r[ix["Address"]][-5:] + " " + " ".join(f"{f(r, c):.3g}" for c in cols) + "  " +
                  r[ix["Source"]].strip()[:70])


if __name__ == "__main__":
    main()
