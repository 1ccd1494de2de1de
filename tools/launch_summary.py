"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv): per kernel name, launches,
total and mean duration, share of the listed GPU time. Usage: python tools/launch_summary.py FILE.csv"""
import csv
import io
import sys
from collections import defaultdict

text = open(sys.argv[1]).read()
rows = list(csv.DictReader(io.StringIO(text[text.index('"ID"'):])))
tot = defaultdict(float)
cnt = defaultdict(int)
for r in rows:
    if r["Metric Name"] != "gpu__time_duration.sum":
        continue
    name = r["Kernel Name"].split("(")[0][:90]
    tot[name] += float(r["Metric Value"].replace(",", "")) * (1e-3 if r["Metric Unit"] == "ns" else 1.0)
    cnt[name] += 1
all_us = sum(tot.values())
print(f"| kernel | launches | total ms | mean us | share |\n|---|---|---|---|---|")
for k in sorted(tot, key=tot.get, reverse=True):
    print(f"| `{k}` | {cnt[k]} | {tot[k] / 1e3:.2f} | {tot[k] / cnt[k]:.1f} | {tot[k] / all_us:.1%} |")
print(f"\n{sum(cnt.values())} launches, {all_us / 1e3:.2f} ms of kernel time (cold-cache, serialised).")
