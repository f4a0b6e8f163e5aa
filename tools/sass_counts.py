"""Per-kernel SASS instruction-class counts of libduet.so: proves which kernels
issue Blackwell tensor-core / TMA / TMEM instructions without a rebuild.

    python tools/sass_counts.py > profiles/r2_sass_counts.md
"""
import collections
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_ipps_zhanghl21_b200", "libduet.so")
CLASSES = [  # (column, regex on the opcode)
    ("UTCHMMA", r"^UTCHMMA$"), ("UTCHMMA.2CTA", r"^UTCHMMA\..*2CTA"), ("UTC*MMA other", r"^UTC[A-Z]*MMA"),
    ("UTCBAR", r"^UTCBAR"), ("LDTM", r"^LDTM"), ("STTM", r"^STTM"), ("UTMALDG", r"^UTMALDG"),
    ("UTMASTG", r"^UTMASTG"), ("UTMAPF", r"^UTMAPF"), ("UBLKCP", r"^UBLKCP"), ("SYNCS", r"^SYNCS"),
    ("HMMA (legacy)", r"^HMMA"), ("FFMA", r"^FFMA"), ("MUFU", r"^MUFU"), ("LDG", r"^LDG"), ("STG", r"^STG"),
]


def demangle(names):
    r = subprocess.run(["c++filt"], input="\n".join(names), capture_output=True, text=True)
    return r.stdout.splitlines() if r.returncode == 0 else names


def main():
    out = subprocess.run(["cuobjdump", "-sass", LIB], capture_output=True, text=True, check=True).stdout
    funcs = collections.OrderedDict()
    cur = None
    for ln in out.splitlines():
        m = re.match(r"\s*Function : (\S+)", ln)
        if m:
            cur = m.group(1)
            funcs[cur] = collections.Counter()
            continue
        m = re.match(r"\s*/\*[0-9a-f]{4,}\*/\s+(?:@!?U?P\w+\s+)?([A-Z][A-Z0-9_.]*)", ln)
        if m and cur:
            op = m.group(1)
            for col, rx in CLASSES:
                if re.search(rx, op) or (col == "UTCHMMA" and op.startswith("UTCHMMA") and "2CTA" not in op):
                    funcs[cur][col] += 1
                    break
    names = demangle(list(funcs))
    print("# SASS instruction classes per kernel (`cuobjdump -sass libduet.so`, `tools/sass_counts.py`)\n")
    print("Counts are static instructions in each kernel's SASS (all template instances summed by base name).\n")
    agg = collections.OrderedDict()
    for mangled, dem in zip(funcs, names):
        base = re.sub(r"<.*", "", dem).replace("duet::(anonymous namespace)::", "").replace("duet::", "")
        agg.setdefault(base, collections.Counter()).update(funcs[mangled])
    cols = [c for c, _ in CLASSES]
    print("| kernel | " + " | ".join(cols) + " |")
    print("|---|" + "---|" * len(cols))
    for base, c in sorted(agg.items()):
        print(f"| `{base}` | " + " | ".join(str(c.get(k, 0)) for k in cols) + " |")


if __name__ == "__main__":
    sys.exit(main())
