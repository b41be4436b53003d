"""Summarise an `ncu --metrics gpu__time_duration.sum --csv` launch list per kernel."""
import collections
import csv
import io
import sys


def load(path):
    lines = [l for l in open(path) if not l.startswith("==")]
    rows = list(csv.reader(io.StringIO("".join(lines))))
    hdr = rows[0]
    ki, vi, ui = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    out = []
    for r in rows[1:]:
        if len(r) <= vi:
            continue
        v = float(r[vi].replace(",", ""))
        v *= {"ns": 1e-3, "nsecond": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3,
              "s": 1e6, "second": 1e6}.get(r[ui].strip(), 1e-3)
        out.append((r[ki], v))
    return out


def short(name):
    n = name.split("(")[0]
    for key in ("gemm_bf16_tc_kernel", "attn_tc_kernel", "layernorm_kernel", "ramp_bert_kernel",
                "compact_kernel", "ring_pop_kernel", "ring_push_kernel"):
        if key in name:
            return key + (name[name.find("<"):name.find(">") + 1] if "<" in name else "")
    return n[:60]


if __name__ == "__main__":
    d = collections.defaultdict(list)
    for k, v in load(sys.argv[1]):
        d[short(k)].append(v)
    tot = sum(sum(v) for v in d.values())
    print(f"{'kernel':44s} {'launches':>8s} {'avg_us':>9s} {'total_us':>10s} {'share':>6s}")
    for k, v in sorted(d.items(), key=lambda kv: -sum(kv[1])):
        print(f"{k:44s} {len(v):8d} {sum(v)/len(v):9.2f} {sum(v):10.1f} {sum(v)/tot:6.3f}")
