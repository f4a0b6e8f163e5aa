"""Summarise an ncu launch list (tools/launch_list.py) into profiles/<tag>_launches.md: per kernel,
launches, summed serialised time and share of the step.

    python tools/launch_md.py r2 c5 gpurun_out/r2_launches_c5.csv 3
"""
import collections
import csv
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def main():
    tag, cfg, path, steps = sys.argv[1], sys.argv[2], sys.argv[3], int(sys.argv[4])
    rows = list(csv.reader(open(path)))
    hdr = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
    h = rows[hdr]
    agg = collections.OrderedDict()
    total = 0.0
    n = 0
    for r in rows[hdr + 1:]:
        if len(r) != len(h):
            continue
        d = dict(zip(h, r))
        if d["Metric Name"] != "gpu__time_duration.sum":
            continue
        v = float(d["Metric Value"].replace(",", ""))
        unit = d.get("Metric Unit", "ns")
        ns = v * {"ns": 1, "nsecond": 1, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6}.get(unit, 1)
        name = re.sub(r"\(.*", "", d["Kernel Name"]).replace("void ", "").replace("duet::(anonymous namespace)::", "")
        name = re.sub(r"duet::<unnamed>::", "", name)
        a = agg.setdefault(name, [0, 0.0])
        a[0] += 1
        a[1] += ns
        total += ns
        n += 1
    out = [f"# {tag}: ncu launch list of {steps} DUET steps of {cfg}", "",
           f"`ncu --metrics gpu__time_duration.sum --clock-control none --profile-from-start off` around "
           f"`tools/launch_list.py {cfg} {steps}` (cudaProfilerStart/Stop bracket the steps).  ncu "
           f"serialises every launch and starts it cold, so the sum ({total / 1e3 / steps:.1f} us per step) "
           f"exceeds the concurrent step; the shares are the check on bench.py's dominant kernel.", "",
           f"{n} launches = {n / steps:.0f} per step.", "",
           "| kernel | launches per step | us per step (serialised) | share |", "|---|---|---|---|"]
    for name, (cnt, ns) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        out.append(f"| `{name}` | {cnt / steps:.0f} | {ns / 1e3 / steps:.1f} | {100 * ns / total:.1f}% |")
    open(os.path.join(ROOT, "profiles", f"{tag}_launches_{cfg}.md"), "w").write("\n".join(out) + "\n")
    print("\n".join(out))


if __name__ == "__main__":
    main()
