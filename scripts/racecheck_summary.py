"""Aggregate compute-sanitizer racecheck output (stdin) by hazard kind and
the (writer, reader) code locations: one line per distinct pair."""
import collections
import re
import sys

cnt = collections.Counter()
kind = None
w = r = None
total = None
for line in sys.stdin:
    m = re.search(r"Error: Potential (\w+) hazard detected \(([^)]*)\)", line)
    if m:
        kind, w, r = f"{m.group(1)} ({m.group(2)})", None, None
        continue
    m = re.search(r"(Write|Read) Thread .*? at (.*)$", line)
    if m and kind:
        loc = re.sub(r"\(CUtensorMap_st.*", "", m.group(2))
        loc = re.sub(r"\+0x[0-9a-f]+", "", loc).strip()
        if m.group(1) == "Write":
            w = loc
        else:
            r = loc
        if w and r:
            cnt[(kind, w, r)] += 1
            kind = None
    if "RACECHECK SUMMARY" in line or "ERROR SUMMARY" in line:
        total = line.strip()
for (k, w, r), n in cnt.most_common():
    print(f"{n:7d}  {k}\n         W: {w}\n         R: {r}")
print(total)
