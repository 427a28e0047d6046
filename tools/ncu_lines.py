"""Per-source-line warp-stall breakdown of one kernel in an ncu report (reads the SASS source page and maps
instruction offsets to lines with nvdisasm -g on the kernel's cubin).

  python tools/ncu_lines.py <report.ncu-rep> <kernel-substring> <cubin-name-substring> <source.cu> [top]
"""
import csv
import io
import os
import re
import subprocess
import sys
import tempfile

LIB = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                   "paper_conf_middleware_hul24_b200", "_lib", "libmenos.so")


def main():
    rep, kern, cub, src = sys.argv[1:5]
    top = int(sys.argv[5]) if len(sys.argv) > 5 else 30
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "-k",
                          f"regex:{kern}"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hi = next(i for i, r in enumerate(rows) if "Address" in r and "Source" in r)
    h = rows[hi]
    i_all = h.index("Warp Stall Sampling (All Samples)")
    reasons = [c for c in h if c.startswith("stall_") and "Not Issued" not in c]
    idx = {c: h.index(c) for c in reasons}
    data = [r for r in rows[hi + 1:] if len(r) > i_all and r[0].startswith("0x")]
    start = int(data[0][0], 16)
    with tempfile.TemporaryDirectory() as d:
        subprocess.run(["cuobjdump", "-xelf", "all", LIB], cwd=d, capture_output=True)
        cubin = next(os.path.join(d, f) for f in os.listdir(d) if cub in f)
        sass = subprocess.run(["nvdisasm", "-g", "-c", cubin], capture_output=True, text=True).stdout
    # nvdisasm -g prints every function; keep the one with the kernel name
    off2line, cur, infn = {}, None, False
    for ln in sass.splitlines():
        if ".text." in ln and ":" in ln:
            infn = kern in ln
        m = re.search(r'line (\d+)', ln)
        if "//##" in ln and m:
            cur = int(m.group(1))
            continue
        m2 = re.search(r'/\*([0-9a-f]{4,})\*/', ln)
        if infn and m2 and cur is not None:
            off2line[int(m2.group(1), 16)] = cur
    agg, per = {}, {}
    for r in data:
        line = off2line.get(int(r[0], 16) - start, -1)
        s = int(r[i_all] or 0)
        agg[line] = agg.get(line, 0) + s
        pr = per.setdefault(line, {})
        for c in reasons:
            v = r[idx[c]]
            if v and v.replace(".", "").isdigit():
                pr[c] = pr.get(c, 0) + float(v)
    tot = sum(agg.values()) or 1
    lines = open(src).read().split("\n")
    for line, s in sorted(agg.items(), key=lambda x: -x[1])[:top]:
        txt = lines[line - 1].strip()[:70] if 0 < line <= len(lines) else "?"
        rs = sorted(per[line].items(), key=lambda x: -x[1])[:3]
        print(f"{s:6d} {100 * s / tot:5.1f}% L{line:<4d} {txt:70s} " + " ".join(f"{k[6:]}={int(v)}" for k, v in rs))


if __name__ == "__main__":
    main()
