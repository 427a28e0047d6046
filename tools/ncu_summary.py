"""Summarise ncu outputs into profiles/ (launch shares of one bench step; per-kernel full-set metrics).

  python tools/ncu_summary.py launches <launches.csv> <launches_per_step> <out.json>
  python tools/ncu_summary.py report <prof.ncu-rep> <out.json>
"""
import csv
import json
import re
import subprocess
import sys
from collections import OrderedDict, defaultdict


def short(name):
    n = re.sub(r"\(.*", "", name)
    n = n.replace("menos::", "").replace("(anonymous namespace)::", "").replace("<unnamed>::", "")
    return n.strip()


def launches(path, per_step, out):
    rows = []
    with open(path) as fh:
        lines = [l for l in fh if l.startswith('"')]
    rd = csv.DictReader(lines)
    for r in rd:
        if r["Metric Name"] == "gpu__time_duration.sum":
            rows.append((r["Kernel Name"], float(r["Metric Value"]), r["Grid Size"], r["Block Size"]))
    last = rows[-per_step:]
    agg = defaultdict(lambda: [0, 0.0])
    for name, ns, g, b in last:
        k = short(name)
        agg[k][0] += 1
        agg[k][1] += ns
    tot = sum(v[1] for v in agg.values())
    res = OrderedDict(sorted(((k, {"launches": v[0], "ms": v[1] / 1e6, "share": v[1] / tot}) for k, v in agg.items()),
                             key=lambda kv: -kv[1]["ms"]))
    doc = {"source": path, "launches_in_step": len(last), "total_ms_serialised": tot / 1e6, "kernels": res,
           "note": "ncu --metrics gpu__time_duration.sum --clock-control none: cold-cache, serialised launches; "
                   "compare SHARES with bench.py's live CUDA-event kernel table, not absolutes"}
    json.dump(doc, open(out, "w"), indent=1)
    for k, v in res.items():
        print(f"{k:60s} {v['launches']:5d} {v['ms']:9.3f} ms {100 * v['share']:5.1f}%")


METRICS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
           "sm__pipe_tensor_op_hmma_cycles_active.avg.pct_of_peak_sustained_active",
           "sm__inst_executed_pipe_tc.avg.pct_of_peak_sustained_active",
           "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
           "launch__registers_per_thread", "launch__grid_size", "sm__warps_active.avg.pct_of_peak_sustained_active",
           "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_bytes.sum", "sm__cycles_elapsed.avg.per_second",
           "sm__ops_path_tensor_op_utchmma_src_bf16_dst_fp32_sparsity_off.avg.pct_of_peak_sustained_elapsed",
           "lts__t_sector_hit_rate.pct", "smsp__inst_executed.sum"]


def report(path, out):
    txt = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    lines = [l for l in txt.splitlines() if l.startswith('"')]
    rd = list(csv.reader(lines))
    hdr = rd[0]
    units = rd[1]
    res = []
    for r in rd[2:]:
        d = dict(zip(hdr, r))
        e = OrderedDict()
        e["kernel"] = short(d.get("Kernel Name", ""))
        e["grid"] = d.get("Grid Size")
        for m in METRICS:
            for col in hdr:
                if col == m:
                    u = units[hdr.index(col)]
                    try:
                        e[m] = float(d[col].replace(",", ""))
                    except ValueError:
                        e[m] = d[col]
                    e[m + "_unit"] = u
        res.append(e)
    json.dump(res, open(out, "w"), indent=1)
    for e in res:
        print(e["kernel"][:40], e.get("grid"), {k: e[k] for k in e if k in METRICS[:4]})


if __name__ == "__main__":
    if sys.argv[1] == "launches":
        launches(sys.argv[2], int(sys.argv[3]), sys.argv[4])
    else:
        report(sys.argv[2], sys.argv[3])
