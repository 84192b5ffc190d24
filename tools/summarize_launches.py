"""Aggregate an `ncu --csv --log-file` launch list per kernel (times, shares,
dram bytes per launch if collected).  Usage: summarize_launches.py in.csv out.txt "title" """
import collections
import csv
import sys


def summarize(path, out, title):
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    hdr = rows[0]
    ki, vi, ui, mi = (hdr.index(k) for k in ("Kernel Name", "Metric Value", "Metric Unit", "Metric Name"))
    agg = collections.defaultdict(lambda: collections.defaultdict(float))
    cnt = collections.Counter()
    for r in rows[1:]:
        v = float(r[vi].replace(",", ""))
        u, name = r[ui], r[mi]
        if name == "gpu__time_duration.sum":
            v = {"ns": 1e-6, "nsecond": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1.0, "ms": 1.0}.get(u, 1.0) * v
            cnt[r[ki]] += 1
        elif "bytes" in name:
            v *= {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
        agg[r[ki]][name] += v
    tot = sum(a["gpu__time_duration.sum"] for a in agg.values())
    with open(out, "w") as f:
        f.write(title + "\ncold-cache, serialised launch times (compare shares, not absolutes)\n\n")
        for k, a in sorted(agg.items(), key=lambda x: -x[1]["gpu__time_duration.sum"]):
            n = cnt[k]
            ms = a["gpu__time_duration.sum"]
            extra = ""
            if "dram__bytes_read.sum" in a:
                extra = (f"  dram R {a['dram__bytes_read.sum'] / n / 1e9:.3f} GB W "
                         f"{a['dram__bytes_write.sum'] / n / 1e9:.3f} GB per launch")
            f.write(f"{n:5d} launches {ms:10.3f} ms {100 * ms / tot:6.2f}%  avg {ms / n:.4f} ms{extra}  {k[:90]}\n")
    return open(out).read()


if __name__ == "__main__":
    print(summarize(sys.argv[1], sys.argv[2], sys.argv[3]))
