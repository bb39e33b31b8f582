"""Executed SASS opcode mix per DP cell from an ncu report with source counters (the
`--set full --import-source on` captures of tools/gpu_run.sh): lane-instructions per cell by
opcode, i.e. the measured counterpart of the per-cell operation counts in DESIGN.md.
usage: python tools/sass_mix.py report.ncu-rep|source.csv cells [top]
(source.csv: `ncu -i report --page source --csv --print-source sass` output)"""
import collections
import csv
import io
import subprocess
import sys

rep, cells = sys.argv[1], float(sys.argv[2])
top = int(sys.argv[3]) if len(sys.argv) > 3 else 20
if rep.endswith(".csv"):
    out = open(rep).read()
else:
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
lines = out.splitlines()
kname = lines[0].split(",", 1)[1].strip().strip('"') if lines else "?"
rows = list(csv.reader(io.StringIO("\n".join(lines[1:]))))
hdr, data = rows[0], rows[1:]
ie = hdr.index("Thread Instructions Executed")
mix = collections.Counter()
for r in data:
    t = r[1].split()
    if not t:
        continue
    op = (t[1] if t[0].startswith("@") else t[0]).split(".")
    name = op[0] + ("." + op[1] if len(op) > 1 and op[0] in ("VIADDMNMX", "VIMNMX", "VIMNMX3", "VIADD") else "")
    mix[name] += int(r[ie] or 0)
tot = sum(mix.values())
print("# executed lane-instructions per cell: %s\n" % kname)
print("cells per launch: %.4g; all opcodes: %.3f lane-instructions per cell\n" % (cells, tot / cells))
print("| opcode | lane-instructions / cell | share |\n|---|---|---|")
for k, v in mix.most_common(top):
    print("| %s | %.4f | %.1f%% |" % (k, v / cells, 100.0 * v / tot))
