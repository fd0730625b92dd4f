"""Summarise the isolated ncu --set full captures (tools/ncu_kernels.sh) into
profiles/r01_ncu_iso_kernels.json: per kernel the launch's duration, DRAM read/write bytes, grid,
registers and the DRAM bytes per element -- the `traffic` that bench.py scales to its own launches.

  python tools/ncu_iso_summary.py gpurun_out profiles/r01_ncu_iso_kernels.json
"""
import csv
import json
import sys

N = 201_379_840
ALG = {"k2_adamw": 30, "k1_cast": 6, "k3_sumsq": 4, "k4_exec_reduce": 12}


def parse(path):
    rows = list(csv.reader(open(path)))
    hdr_i = next(i for i, r in enumerate(rows) if "gpu__time_duration.sum" in r)
    hdr, units, vals = rows[hdr_i], rows[hdr_i + 1], rows[hdr_i + 2]
    out = {}
    for h, u, v in zip(hdr, units, vals):
        try:
            x = float(v.replace(",", ""))
        except ValueError:
            continue
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6,
                 "msecond": 1e-3, "ns": 1e-9, "us": 1e-6, "ms": 1e-3}.get(u, 1)
        out[h] = x * scale
    return out


def main():
    src, dst = sys.argv[1], sys.argv[2]
    res = {"n_elements": N, "source": "ncu --set full --clock-control none, tools/ncu_kernels.sh (isolated, one launch)"}
    for k, alg in ALG.items():
        try:
            m = parse(f"{src}/ncu_iso_{k}.csv")
        except Exception as e:  # noqa: BLE001
            res[k] = {"error": str(e)}
            continue
        rd, wr, t = m.get("dram__bytes_read.sum"), m.get("dram__bytes_write.sum"), m.get("gpu__time_duration.sum")
        res[k] = {"duration_s": t, "dram_read_bytes": rd, "dram_write_bytes": wr,
                  "dram_bytes_per_elem": (rd + wr) / N, "algorithmic_bytes_per_elem": alg,
                  "traffic_over_algorithmic": (rd + wr) / (alg * N),
                  "achieved_alg_gbs": alg * N / t / 1e9,
                  "grid": m.get("launch__grid_size"), "regs": m.get("launch__registers_per_thread")}
    json.dump(res, open(dst, "w"), indent=1)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
