"""Summarise `ncu --set full` raw CSVs into profiles/<tag>_full.md and profiles/ncu_summary.json
(read by bench.py for roofline.traffic: DRAM bytes per launch of each config's dominant kernel).

    python tools/full_md2.py r2 c5:b4_gru=gpurun_out/r2_full_gru1024_raw.csv ...
    python tools/full_md2.py r2_tf32 --no-summary fc1_f32=gpurun_out/...raw.csv   (md only)
"""
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3,
        "nsecond": 1e-3, "msecond": 1e3, "%": 1.0, "": 1.0}
KEYS = [("gpu__time_duration.sum", "duration (us)"), ("dram__bytes_read.sum", "DRAM read (B)"),
        ("dram__bytes_write.sum", "DRAM write (B)"),
        ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed", "tensor pipe active % (elapsed)"),
        ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "tensor pipe active % (active)"),
        ("l1tex__m_xbar2l1tex_read_bytes_mem_global_op_tma_ld.sum", "TMA bytes read (B)"),
        ("launch__grid_size", "grid"), ("launch__registers_per_thread", "registers / thread")]


def read(path):
    rows = list(csv.reader(open(path)))
    h, units, v = rows[0], rows[1], rows[2]
    out = {"kernel": v[h.index("Kernel Name")]}
    for k, _ in KEYS:
        if k in h:
            i = h.index(k)
            try:
                out[k] = float(v[i].replace(",", "")) * UNIT.get(units[i], 1.0)
            except ValueError:
                out[k] = None
    return out


def main():
    args = [a for a in sys.argv[1:] if a != "--no-summary"]
    tag = args[0]
    items = [a.split("=", 1) for a in args[1:]]
    lines = [f"# {tag}: `ncu --set full --clock-control none` captures (one launch each, cold-cache replay)", ""]
    summary = {"tag": tag, "kernels": {}}
    for name, path in items:
        d = read(path)
        lines += [f"## {name}", "", f"`{d['kernel'][:160]}`", "", "| metric | value |", "|---|---|"]
        for k, label in KEYS:
            if k in d and d[k] is not None:
                lines.append(f"| {label} (`{k}`) | {d[k]:.6g} |")
        lines.append("")
        summary["kernels"][name] = {"dram_bytes": (d.get("dram__bytes_read.sum") or 0) + (d.get("dram__bytes_write.sum") or 0),
                                    "ncu_duration_us": d.get("gpu__time_duration.sum"),
                                    "tensor_pipe_pct": d.get("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed"),
                                    "kernel": d["kernel"][:120]}
    open(os.path.join(ROOT, "profiles", f"{tag}_full.md"), "w").write("\n".join(lines) + "\n")
    if "--no-summary" not in sys.argv:  # (extra captures: keep bench.py's per-config summary)
        json.dump(summary, open(os.path.join(ROOT, "profiles", "ncu_summary.json"), "w"), indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
