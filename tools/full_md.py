"""profiles/<tag>_full.md from `ncu --page raw --csv` exports of single-kernel full captures.
  python tools/full_md.py r1c name:description:raw.csv ..."""
import csv
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "DRAM read"),
    ("dram__bytes_write.sum", "DRAM write"),
    ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed", "tensor pipe active %"),
    ("sm__throughput.avg.pct_of_peak_sustained_elapsed", "SM throughput %"),
    ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "DRAM throughput %"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "L2 throughput %"),
    ("launch__registers_per_thread", "registers/thread"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps active %"),
]


def main():
    tag = sys.argv[1]
    out = [f"# {tag}: `ncu --set full --clock-control none` captures (one launch each, cold-cache replay)", "",
           f"Commands: `tools/ncu_round.sh {tag}` on the B200 (gpurun).  Raw CSVs: `profiles/{tag}_*_raw.csv`.", ""]
    for spec in sys.argv[2:]:
        name, desc, path = spec.split(":", 2)
        rows = list(csv.reader(open(path)))
        hdr, units = rows[0], rows[1]
        val = rows[2]
        d = dict(zip(hdr, val))
        u = dict(zip(hdr, units))
        out += [f"## {name}: {desc}", "", f"`{d.get('Kernel Name', '?')[:140]}` grid {d.get('Grid Size', '?')} "
                f"block {d.get('Block Size', '?')}", "", "| metric | value |", "|---|---|"]
        for m, label in METRICS:
            if m in d:
                out.append(f"| {label} (`{m}`) | {d[m]} {u.get(m, '')} |")
        out.append("")
    with open(os.path.join(ROOT, "profiles", f"{tag}_full.md"), "w") as f:
        f.write("\n".join(out) + "\n")


if __name__ == "__main__":
    main()
