"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) by kernel name.

usage: python tools/launch_summary.py LAUNCHES.csv > profiles/..._launch_summary.txt
"""
import collections
import csv
import sys

rows = [r for r in csv.reader(l for l in open(sys.argv[1]) if l.startswith('"'))]
hdr = rows[0]
iN, iV = hdr.index("Kernel Name"), hdr.index("Metric Value")
tot = collections.defaultdict(float)
cnt = collections.Counter()
for r in rows[1:]:
    name = r[iN].split("(")[0]
    tot[name] += float(r[iV].replace(",", "")) / 1e6
    cnt[name] += 1
allms = sum(tot.values())
print(f"# {sys.argv[1]}: {sum(cnt.values())} launches, {allms:.2f} ms total (cold-cache, serialised by ncu)")
for name, ms in sorted(tot.items(), key=lambda x: -x[1]):
    print(f"{ms:10.3f} ms {100 * ms / allms:6.2f}%  x{cnt[name]:<4d} {name}")
