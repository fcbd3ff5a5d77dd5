"""Per-function warp-stall reasons from an ncu --set full report's source page:
python tools/ncu_stalls_by_function.py REPORT.ncu-rep [reason ...] (default: no_inst long_sb wait)"""
import csv
import io
import subprocess
import sys

sys.path.insert(0, __import__("os").path.dirname(__file__))
from ncu_by_function import function_starts  # noqa: E402

rep = sys.argv[1]
reasons = ["stall_" + r for r in (sys.argv[2:] or ["no_inst", "long_sb", "wait", "branch_resolving"])]
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(src)))
hdr = next(r for r in rows if r and r[0] == "Line No")
idx = {c: hdr.index(c) for c in reasons + ["Warp Stall Sampling (All Samples)", "Instructions Executed"]}
starts = function_starts()
agg, tot = {}, {c: 0 for c in idx}
for r in rows:
    if not r or r[0] in ("", "Line No"):
        continue
    try:
        ln = int(r[0])
    except ValueError:
        continue
    fn = "?"
    for s, n in starts:
        if s <= ln:
            fn = n
        else:
            break
    a = agg.setdefault(fn, {c: 0 for c in idx})
    for c, i in idx.items():
        try:
            v = int(float(r[i].replace(",", ""))) if r[i] not in ("", "-") else 0
        except ValueError:
            v = 0
        a[c] += v
        tot[c] += v
key = "Warp Stall Sampling (All Samples)"
print(f"# {rep}: share of each column per function")
print(f"{'function':22s} {'samples':>8s} {'instr':>7s} " + " ".join(f"{c[6:]:>9s}" for c in reasons))
for fn, a in sorted(agg.items(), key=lambda x: -x[1][key])[:25]:
    print(f"{fn:22s} {100 * a[key] / tot[key]:7.1f}% {100 * a['Instructions Executed'] / tot['Instructions Executed']:6.1f}% "
          + " ".join(f"{100 * a[c] / max(1, tot[c]):8.1f}%" for c in reasons))
