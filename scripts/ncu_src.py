"""Per-source-line instructions executed and stall samples from an ncu report (needs -lineinfo).

    python scripts/ncu_src.py report.ncu-rep [top]
"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
k = int(sys.argv[2]) if len(sys.argv) > 2 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda"],
                     capture_output=True, text=True).stdout
blocks = out.split('"Kernel Name"')
for b in blocks[1:]:
    lines = b.split("\n")
    rows = list(csv.reader(io.StringIO("\n".join(lines[1:]))))
    hdr = rows[0]
    ie = hdr.index("Instructions Executed") if "Instructions Executed" in hdr else None
    si = hdr.index("Warp Stall Sampling (All Samples)")
    src = hdr.index("Source")
    ln = hdr.index("#") if "#" in hdr else 0
    data = []
    for r in rows[1:]:
        if len(r) <= si:
            continue
        try:
            data.append((int(r[ie] or 0) if ie is not None else 0, int(r[si] or 0), r[ln], r[src].strip()))
        except ValueError:
            pass
    ti = sum(d[0] for d in data) or 1
    ts = sum(d[1] for d in data) or 1
    print("==", lines[0][:100], "inst", ti, "samples", ts)
    for d in sorted(data, key=lambda d: -d[0])[:k]:
        print(f"inst {d[0] / ti:6.3f} stall {d[1] / ts:6.3f}  L{d[2]:>5s}  {d[3][:100]}")
