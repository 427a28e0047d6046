"""Per-GEMM DRAM traffic of one cfg1 layer against its algorithmic bytes.

  ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum -k regex:gemm_tc_kernel \
      -s 24 -c 8 --csv python bench.py --layers 1 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gemm.csv
  python tools/gemm_traffic.py gemm.csv profiles/gemm_traffic.json

The 8 launches after the 3 warm-up steps are one layer's forward (QKV+RoPE, O+resid, gate|up+SwiGLU, down+resid)
and backward (down-dX+SwiGLU-bwd, gate|up-dX, O-dX+rowsum, QKV-dX).  Algorithmic bytes = operands read once + outputs
written once (cfg1: T = 8192, d = 4096, f = 11008, H = 32; bf16 operands, fp32 residual stream; the small LoRA
extra-K window is ignored)."""
import csv
import io
import json
import sys

T, d, f, H = 8192, 4096, 11008, 32
ALG = {   # name: bytes
    "fwd QKV (+RoPE)": 2 * (T * d + 3 * d * d + 3 * T * d),
    "fwd O (+resid fp32)": 2 * T * d + 2 * d * d + 8 * T * d,
    "fwd gate|up (+SwiGLU)": 2 * T * d + 4 * f * d + 4 * T * f + 2 * T * f,
    "fwd down (+resid fp32)": 2 * T * f + 2 * d * f + 8 * T * d,
    "bwd down-dX (+SwiGLU-bwd)": 2 * T * d + 2 * d * f + 4 * T * f + 4 * T * f,
    "bwd gate|up-dX": 4 * T * f + 4 * f * d + 2 * T * d,
    "bwd O-dX (+rowsum)": 2 * T * d + 2 * d * d + 2 * T * d + 2 * T * d + 4 * H * T,
    "bwd QKV-dX": 6 * T * d + 6 * d * d + 2 * T * d,
}


def main():
    src, out = sys.argv[1], sys.argv[2]
    text = open(src).read()
    rows = list(csv.reader(io.StringIO(text[text.index('"ID"'):])))
    h = rows[0]
    iid, iname, ival = h.index("ID"), h.index("Metric Name"), h.index("Metric Value")
    per = {}
    for r in rows[1:]:
        if len(r) <= ival:
            continue
        per.setdefault(int(r[iid]), {})[r[iname]] = float(r[ival].replace(",", ""))
    launches = [per[k] for k in sorted(per)][:8]
    res = []
    for (name, alg), m in zip(ALG.items(), launches):
        dram = m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)
        res.append({"gemm": name, "algorithmic_bytes": alg, "dram_bytes": dram, "ratio": dram / alg,
                    "ms": m.get("gpu__time_duration.sum", 0) / 1e6})
    mean = sum(r["dram_bytes"] for r in res) / max(len(res), 1)
    json.dump({"source": "ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum (one cfg1 layer, 8 GEMMs)",
               "per_gemm": res, "bytes_per_launch": mean}, open(out, "w"), indent=1)
    for r in res:
        print(f'{r["gemm"]:28s} dram {r["dram_bytes"] / 1e6:8.1f} MB  alg {r["algorithmic_bytes"] / 1e6:8.1f} MB  '
              f'x{r["ratio"]:.2f}  {r["ms"]:.3f} ms')


if __name__ == "__main__":
    main()
