"""Summarise an ncu launch list (--metrics gpu__time_duration.sum[,dram__bytes_read.sum,dram__bytes_write.sum]
--csv): per kernel the launch count, mean / total duration, share of the total,
and mean DRAM bytes per launch.

    python scripts/ncu_launch_summary.py launches.csv [out.txt]
"""
import csv
import re
import sys
from collections import OrderedDict, defaultdict

SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-3, "usecond": 1.0, "msecond": 1e3,
         "ns": 1e-3, "us": 1.0, "ms": 1e3}


def short(name):
    n = re.sub(r"\(.*", "", name)
    n = n.replace("void ", "").replace("e3::<unnamed>::", "").replace("(anonymous namespace)::", "")
    return n.strip()


def main(path, out=None):
    rows = [r for r in csv.reader(l for l in open(path) if not l.startswith("=="))]
    h = rows[0]
    ki, mi, vi, ui, ii = (h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"),
                          h.index("Metric Unit"), h.index("ID"))
    launches = OrderedDict()
    for r in rows[1:]:
        d = launches.setdefault(r[ii], {"k": short(r[ki])})
        try:
            d[r[mi]] = float(r[vi].replace(",", "")) * SCALE.get(r[ui], 1.0)
        except ValueError:
            pass
    agg = defaultdict(lambda: [0, 0.0, 0.0, 0.0])
    for d in launches.values():
        a = agg[d["k"]]
        a[0] += 1
        a[1] += d.get("gpu__time_duration.sum", 0.0)
        a[2] += d.get("dram__bytes_read.sum", 0.0)
        a[3] += d.get("dram__bytes_write.sum", 0.0)
    tot = sum(a[1] for a in agg.values())
    lines = [f"{'kernel':48s} {'launches':>8s} {'avg_us':>9s} {'total_us':>11s} {'share':>6s} "
             f"{'dram_rd_MB':>10s} {'dram_wr_MB':>10s}"]
    for k, a in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        lines.append(f"{k[:48]:48s} {a[0]:8d} {a[1] / a[0]:9.2f} {a[1]:11.1f} {a[1] / tot:6.3f} "
                     f"{a[2] / a[0] / 1e6:10.2f} {a[3] / a[0] / 1e6:10.2f}")
    lines.append(f"total {tot:.1f} us over {len(launches)} launches")
    txt = "\n".join(lines)
    print(txt)
    if out:
        open(out, "w").write(txt + "\n")


if __name__ == "__main__":
    main(*sys.argv[1:])
