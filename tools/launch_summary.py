"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) into a markdown table of
per-kernel launches, total time and share.  usage: python tools/launch_summary.py launches.csv [title]"""
import csv
import collections
import io
import sys

text = open(sys.argv[1]).read()
start = text.find('"ID"')
rows = list(csv.DictReader(io.StringIO(text[start:])))
tot = collections.defaultdict(float)
cnt = collections.Counter()
for r in rows:
    if r.get("Metric Name") != "gpu__time_duration.sum":
        continue
    v = float(r["Metric Value"].replace(",", ""))
    unit = r.get("Metric Unit", "")
    ms = v / 1e6 if unit == "nsecond" else v / 1e3 if unit == "usecond" else v if unit == "msecond" else v / 1e6
    name = r["Kernel Name"].split("(")[0][:70]
    tot[name] += ms
    cnt[name] += 1
allms = sum(tot.values())
title = sys.argv[2] if len(sys.argv) > 2 else sys.argv[1]
print("# ncu launch list: %s\n" % title)
print("Cold-cache, serialised launches (compare SHARES, not absolutes).\n")
print("| kernel | launches | total ms | share |\n|---|---|---|---|")
for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
    print("| %s | %d | %.3f | %.1f%% |" % (k, cnt[k], v, 100 * v / allms))
