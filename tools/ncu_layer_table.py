"""Per-kernel totals from an ncu --csv metrics log (gpu__time_duration.sum, dram__bytes_*), divided by a pass count.

  python tools/ncu_layer_table.py <ncu.csv> [passes]
"""
import csv
import sys


def main():
    path = sys.argv[1]
    passes = int(sys.argv[2]) if len(sys.argv) > 2 else 1
    rows = [r for r in csv.reader(open(path)) if len(r) > 14 and r[0].isdigit()]
    per = {}
    for r in rows:
        per.setdefault(int(r[0]), {"k": r[4].split("(")[0].replace("void ", "").replace("unnamed>::", ""),
                                   "grid": r[8]})[r[12]] = float(r[14])
    agg = {}
    for _, v in sorted(per.items()):
        a = agg.setdefault(v["k"], [0, 0.0, 0.0])
        a[0] += 1
        a[1] += v.get("gpu__time_duration.sum", 0) / 1e3
        a[2] += (v.get("dram__bytes_read.sum", 0) + v.get("dram__bytes_write.sum", 0)) / 1e6
    tot = 0.0
    for k, (n, us, mb) in agg.items():
        tot += us / passes
        print(f"{k:44s} launches={n:4d}  us/pass={us / passes:9.1f}  MB/pass={mb / passes:9.1f}  GB/s={mb / us * 1e3 if us else 0:7.0f}")
    print(f"total us/pass {tot:.1f}")


if __name__ == "__main__":
    main()
