"""Kernel time shares from an ncu launch list (--metrics gpu__time_duration.sum --csv).

ncu serialises and cache-flushes every launch, so absolute times are cold and pessimistic; the
*shares* are what is compared with the bench's CUDA-event view of the step."""
import csv
import re
import sys
from collections import defaultdict


def short(name):
    name = re.sub(r"\(.*", "", name)
    name = name.replace("void ", "").replace("sfs::", "").replace("(anonymous namespace)::", "")
    name = name.replace("<unnamed>::", "")
    return name.strip()


def main(path):
    tot = defaultdict(float)
    cnt = defaultdict(int)
    with open(path) as fh:
        lines = [l for l in fh if l.startswith('"')]
    rows = list(csv.reader(lines))
    h = rows[0]
    ik = h.index("Kernel Name")
    im = h.index("Metric Name")
    iv = h.index("Metric Value")
    for r in rows[1:]:
        if len(r) <= iv or r[im] != "gpu__time_duration.sum":
            continue
        v = float(r[iv].replace(",", ""))
        k = short(r[ik])
        tot[k] += v
        cnt[k] += 1
    allt = sum(tot.values())
    print(f"launches: {sum(cnt.values())}  total kernel time: {allt / 1e6:.3f} ms (ncu units: ns)")
    fam = defaultdict(float)
    for k, v in tot.items():
        base = k.split("<")[0]
        fam[base] += v
    print("by kernel family:")
    for k, v in sorted(fam.items(), key=lambda t: -t[1]):
        print(f"  {100 * v / allt:6.2f}%  {v / 1e6:9.3f} ms  {k}")
    print("by instantiation (top 25):")
    for k, v in sorted(tot.items(), key=lambda t: -t[1])[:25]:
        print(f"  {100 * v / allt:6.2f}%  {v / 1e6:9.3f} ms  {cnt[k]:7d} launches  {k}")


if __name__ == "__main__":
    main(sys.argv[1])
