"""Summarise an ncu launch list (`--metrics gpu__time_duration.sum --csv`) into a
markdown table of per-kernel launches, total and mean time and share.

    python tools/launch_list.py gpurun_out/launches_c2.csv profiles/r1_launches_c2.md "<command line>"
"""
import csv
import io
import sys
from collections import OrderedDict


def main(src, out, cmd):
    text = open(src).read()
    lines = [l for l in text.splitlines() if l.startswith('"')]   # drop ==PROF== lines
    rows = list(csv.DictReader(io.StringIO("\n".join(lines))))
    per = OrderedDict()
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        v = float(r["Metric Value"].replace(",", ""))
        unit = r.get("Metric Unit", "ns")
        us = v / 1e3 if unit in ("ns", "nsecond") else v * 1e3 if unit in ("ms", "msecond") else v
        k = r["Kernel Name"]
        n, t = per.get(k, (0, 0.0))
        per[k] = (n + 1, t + us)
    total = sum(t for _, t in per.values()) or 1.0
    md = ["# timed region of %s (ncu --metrics gpu__time_duration.sum --clock-control none)" % cmd, "",
          "Cold-cache, serialised replay (ncu kernel replay): compare shares, not absolutes.", "",
          "| kernel | launches | total us | mean us | share |", "|---|---|---|---|---|"]
    for k, (n, t) in sorted(per.items(), key=lambda kv: -kv[1][1]):
        md.append("| %s | %d | %.1f | %.1f | %.1f%% |" % (k[:90], n, t, t / n, 100 * t / total))
    open(out, "w").write("\n".join(md) + "\n")
    print("\n".join(md))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], sys.argv[3] if len(sys.argv) > 3 else "bench.py")
