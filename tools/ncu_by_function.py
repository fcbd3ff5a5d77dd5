"""Aggregate an ncu --set full report's source page (warp-stall samples, instructions executed)
per kernel.cu function: python tools/ncu_by_function.py REPORT.ncu-rep [OUT.txt]

Inlined callees keep their own line info, so the totals are per source function (run_jobs,
build_nodes, gather_batch, acquire_work, ...), not per call site."""
import csv
import io
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
SRC = os.path.join(ROOT, "paper_conf_sc_weij22_b200", "csrc", "kernel.cu")


def function_starts():
    pat = re.compile(r"^(?:template.*)?(?:__device__|__global__|static|struct)\b.*?(\w+)\s*\(")
    starts = []
    for i, line in enumerate(open(SRC), 1):
        m = pat.match(line)
        if m and not line.rstrip().endswith(";"):
            starts.append((i, m.group(1)))
    return starts


def main(rep, out=None):
    src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(src)))
    hdr = next(r for r in rows if r and r[0] == "Line No")
    hdr = hdr[:2] + hdr[2:]  # Line No, Source, Address, Source, metrics...
    cols = {name: hdr.index(name) for name in ("Warp Stall Sampling (All Samples)", "Instructions Executed",
                                               "L2 Theoretical Sectors Global Excessive")
            if name in hdr}
    starts = function_starts()
    agg = {}
    tot = {c: 0 for c in cols}
    for r in rows:
        if not r or r[0] in ("", "Line No"):
            continue
        try:
            ln = int(r[0])
        except ValueError:
            continue
        fn = "?"
        for s, name in starts:
            if s <= ln:
                fn = name
            else:
                break
        a = agg.setdefault(fn, {c: 0 for c in cols})
        for c, i in cols.items():
            try:
                v = int(float(r[i].replace(",", ""))) if i < len(r) and r[i] else 0
            except ValueError:
                v = 0
            a[c] += v
            tot[c] += v
    key = "Warp Stall Sampling (All Samples)"
    lines = [f"# per-function totals from {rep} ({', '.join(cols)})"]
    for fn, a in sorted(agg.items(), key=lambda x: -x[1].get(key, 0)):
        parts = [f"{c.split(' (')[0][:22]}={100.0 * a[c] / max(1, tot[c]):5.1f}%" for c in cols]
        lines.append(f"{fn:28s} " + "  ".join(parts))
    text = "\n".join(lines[:40]) + "\n"
    if out:
        open(out, "w").write(text)
    print(text)


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else None)
