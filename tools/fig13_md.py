"""Render tools/fig13.py's JSON as the Fig. 13 table.

  python tools/fig13_md.py gpurun_out/fig13_r1d.json r1d > profiles/r1d_fig13.md"""
import json
import sys

ROWS = [("serial", "Serial (1 stream)"), ("random", "Random (mean 8 seeds)"), ("round_robin", "Round-Robin"),
        ("random_correction", "Random+Correction (mean 8)"), ("greedy", "Greedy (Steps 1-2)"),
        ("greedy_correction", "Greedy+Correction (model Step 3)"),
        ("greedy_correction_measured", "Greedy+Correction (measured Step 3)"),
        ("ideal_model", "Ideal over the model (exhaustive)"), ("ideal_measured", "Ideal measured (exhaustive, D^n<=256)")]


def main():
    res = json.load(open(sys.argv[1]))
    tag = sys.argv[2]
    cfgs = list(res)
    print(f"# Scheduler comparison on B200, {tag} (SURVEY.md §8(f) N2; PAPER.md:88 Fig. 13)\n")
    print(f"`python tools/fig13.py --configs {','.join(cfgs)}` on one B200, 2 stream slots, full sizes, bf16, the library "
          f"at the time of the run (automatic RNN gate-tile width).  Per scheduler: measured p50 of its assignment (ms; CUDA "
          f"events on the home stream, 50 replays, inputs resident, L2 warm) and, in brackets, the C3 model makespan "
          f"from the device profile.  Fallback disabled so every scheduler's own placement runs.  Raw: "
          f"`{tag}_fig13.json`.\n")
    print("| scheduler | " + " | ".join(cfgs) + " |")
    print("|---|" + "---|" * len(cfgs))
    for key, title in ROWS:
        cells = []
        for c in cfgs:
            r = res[c].get(key)
            if r is None:
                cells.append("—")
            elif "model_ms" in r:
                cells.append(f"{r['measured_ms']:.4f} ({r['model_ms']:.4f})")
            else:
                cells.append(f"{r['measured_ms']:.4f}")
        print(f"| {title} | " + " | ".join(cells) + " |")
    print("\nMeasured-Step-3 evaluations: " + ", ".join(
        f"{c} {res[c]['greedy_correction_measured'].get('evaluations')}" for c in cfgs) + ".")


if __name__ == "__main__":
    main()
