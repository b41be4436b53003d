"""Top SASS instructions by warp-stall samples from an ncu report (source page)."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
k = int(sys.argv[2]) if len(sys.argv) > 2 else 25
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
blocks = out.split('"Kernel Name"')
for b in blocks[1:]:
    lines = b.split("\n")
    name = lines[0]
    rows = list(csv.reader(io.StringIO("\n".join(lines[1:]))))
    hdr = rows[0]
    si = hdr.index("Warp Stall Sampling (All Samples)")
    data = [(int(r[si] or 0), r[1].strip()) for r in rows[1:] if len(r) > si]
    tot = sum(d[0] for d in data) or 1
    print("==", name[:100], "total samples", tot)
    for s, ins in sorted(data, key=lambda d: -d[0])[:k]:
        print(f"{s / tot:6.3f}  {ins[:110]}")
