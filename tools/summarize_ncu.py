"""Summarise ncu captures into profiles/ (committed evidence).

    python tools/summarize_ncu.py r1 gpurun_out/launches_r1.csv gpurun_out/fc1_r1_raw.csv

Writes profiles/<tag>_launches.md (per-kernel share of the timed steps' device time from the
cold-cache serialised launch list), profiles/<tag>_fc1.md (key metrics of the dominant kernel's
full capture) and profiles/ncu_summary.json (read by bench.py for roofline.traffic)."""
import collections
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def launches(path):
    rows = list(csv.reader(open(path)))
    hdr = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    h = rows[hdr]
    per = collections.OrderedDict()
    for r in rows[hdr + 1:]:
        if len(r) != len(h):
            continue
        d = dict(zip(h, r))
        key = (d["ID"], d["Kernel Name"], d["Grid Size"], d["Block Size"])
        per.setdefault(key, {})[d["Metric Name"]] = float(d["Metric Value"].replace(",", ""))
    return per


def main():
    tag, launch_csv, full_csv = sys.argv[1:4]
    # optional: a substring of "<kernel> grid<grid>" keys that are not c2 step kernels (e.g. bench.py's
    # secondary roofline launches at B = 65536), listed separately and left out of the step shares
    exclude = sys.argv[4] if len(sys.argv) > 4 else None
    per = launches(launch_csv)
    # the last 3 timed steps: take the launches after the profiler/warm-up (last 3*7 of the bench graph)
    items = list(per.items())
    agg = collections.OrderedDict()
    for (lid, name, grid, block), m in items:
        short = name.split("(")[0].replace("void ", "").replace("unnamed>::", "")
        k = f"{short} grid{grid}"
        a = agg.setdefault(k, {"n": 0, "ns": 0.0, "rd": 0.0, "wr": 0.0})
        a["n"] += 1
        a["ns"] += m.get("gpu__time_duration.sum", 0.0)
        a["rd"] += m.get("dram__bytes_read.sum", 0.0)
        a["wr"] += m.get("dram__bytes_write.sum", 0.0)
    # share of one step: each kernel once (bench.py also launches fc1 alone for the roofline timing)
    extra = collections.OrderedDict((k, agg.pop(k)) for k in list(agg) if exclude and exclude in k)
    tot = sum(a["ns"] / a["n"] for a in agg.values())
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    with open(os.path.join(ROOT, "profiles", f"{tag}_launches.md"), "w") as f:
        f.write(f"# {tag}: ncu launch list (bench.py c2, all launches of our kernels incl. profiling)\n\n")
        f.write("`ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum "
                "--clock-control none` — cold-cache, serialised: compare shares, not absolutes.\n\n")
        f.write("| kernel | launches | mean us | share of a step | mean DRAM read MB | mean DRAM write MB |\n|---|---|---|---|---|---|\n")
        for k, a in sorted(agg.items(), key=lambda kv: -kv[1]["ns"]):
            n = a["n"]
            unit = 1e-3 if a["ns"] / n > 1000 else 1.0  # ncu reports ns or us depending on version
            f.write(f"| {k} | {n} | {a['ns'] / n * (1e-3 if unit == 1e-3 else 1):.2f} | {a['ns'] / n / tot:.1%} | "
                    f"{a['rd'] / n / 1e6:.2f} | {a['wr'] / n / 1e6:.2f} |\n")
        for k, a in extra.items():
            n = a["n"]
            f.write(f"| {k} (not a step kernel: bench.py secondary roofline) | {n} | {a['ns'] / n * (1e-3 if a['ns'] / n > 1000 else 1):.2f} | - | "
                    f"{a['rd'] / n / 1e6:.2f} | {a['wr'] / n / 1e6:.2f} |\n")
    # full capture of the dominant kernel
    r = list(csv.reader(open(full_csv)))
    h = r[0]
    units = dict(zip(h, r[1]))
    keep = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
            "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
            "sm__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
            "lts__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
            "launch__shared_mem_per_block_dynamic", "sm__warps_active.avg.pct_of_peak_sustained_active"]
    caps = []
    for row in r[2:]:
        d = dict(zip(h, row))
        caps.append({k: (d.get(k), units.get(k)) for k in ["Kernel Name", "Grid Size", "Block Size"] + keep})
    with open(os.path.join(ROOT, "profiles", f"{tag}_fc1.md"), "w") as f:
        f.write(f"# {tag}: `ncu --set full` of the c2 GEMMs (gemm2_kernel)\n\n")
        for c in caps:
            f.write(f"## {c['Kernel Name'][0][:80]}  grid {c['Grid Size'][0]} block {c['Block Size'][0]}\n\n")
            for k in keep:
                v, u = c[k]
                f.write(f"- {k}: {v} {u or ''}\n")
            f.write("\n")
    fc1 = next((c for c in caps if "<128" in c["Kernel Name"][0] or c["Grid Size"][0].startswith("(16, 8")), caps[0])

    def mb(v, u):
        x = float(v)
        return x * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1e6)

    dram = mb(*fc1["dram__bytes_read.sum"]) + mb(*fc1["dram__bytes_write.sum"])
    summary = {"tag": tag, "kernels": {"fc1": {"dram_bytes": dram, "ncu_duration": fc1["gpu__time_duration.sum"],
                                                "tensor_pipe_pct": fc1["sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed"][0]}}}
    with open(os.path.join(ROOT, "profiles", "ncu_summary.json"), "w") as f:
        json.dump(summary, f, indent=1)
    print(json.dumps(summary))


if __name__ == "__main__":
    main()
