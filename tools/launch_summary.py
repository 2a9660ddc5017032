"""Summarise an ncu --metrics gpu__time_duration.sum --csv launch list:
launches, total ms and share of the step per kernel (for profiles/)."""
import collections
import csv
import sys

rows = [r for r in csv.reader(open(sys.argv[1])) if r]
hdr = next(i for i, r in enumerate(rows) if "Kernel Name" in r and "Metric Value" in r)
h = rows[hdr]
ki, vi, ui = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
tot = collections.defaultdict(float)
cnt = collections.Counter()
for r in rows[hdr + 1:]:
    if len(r) < len(h):
        continue
    v = float(r[vi].replace(",", ""))
    v = v / 1e6 if r[ui] in ("nsecond", "ns") else (v / 1e3 if r[ui] in ("usecond", "us") else v)
    tot[r[ki]] += v
    cnt[r[ki]] += 1
all_ms = sum(tot.values())
print(sys.argv[2] if len(sys.argv) > 2 else "")
print("(cold-cache, serialised launches under ncu: compare shares, not absolutes)")
print("launches   total ms  share  kernel")
for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
    print(f"{cnt[k]:8d} {v:10.3f} {100 * v / all_ms:5.1f}%  {k[:100]}")
