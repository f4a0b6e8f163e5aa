"""Render tools/sweeps.py's JSON as profiles/<tag>_sweeps.md (§VI-D).

    python tools/sweeps_md.py profiles/r2_sweeps.json r2 > profiles/r2_sweeps.md
"""
import json
import sys


def main():
    d = json.load(open(sys.argv[1]))
    tag = sys.argv[2]
    out = [f"# {tag}: model-variation sweeps on c4 (SURVEY.md §8(f) N3; PAPER.md:89 §VI-D, Figs. 14-17)", "",
           "`python tools/sweeps.py` on one B200 (gpurun): c4 with one dimension varied; 2 CUDA-stream slots, "
           "greedy-correction with measured Step 3 (cold replays, interleaved re-timing of the best candidates), the "
           "recurrence's gate-tile width chosen by measurement (`harness.tuned_session`), p50 of 50 steps (CUDA events "
           f"on the home stream, L2 flushed before every step).  Raw: `profiles/{tag}_sweeps.json`.", ""]
    for key in ("rnn", "cnn", "ffn", "batch"):
        if key not in d:
            continue
        sec = d[key]
        out += [f"## {sec['title']}", "",
                "| variant | p50 DUET (ms) | p50 serial (ms) | speed-up | tile_n kept | profile CNN / RNN / FFN / join (ms) | slots |",
                "|---|---|---|---|---|---|---|"]
        for r in sec["rows"]:
            v = ", ".join(f"{k}={x}" for k, x in r["variant"].items())
            prof = " / ".join(f"{x:.3f}" for x in r["profile_ms"])
            out.append(f"| {v} | {r['p50_ms']:.3f} | {r['serial_p50_ms']:.3f} | {r['speedup_vs_serial']:.2f} | "
                       f"{r['rnn_tile_n']} | {prof} | {r['slot_of']} |")
        out.append("")
    print("\n".join(out))


if __name__ == "__main__":
    main()
