"""Summarise LV_TRACE=2 timelines (tools/trace_run.py, second run): per-level
sweep / modularity / contraction totals and per-class kernel times."""
import re
import sys
from collections import defaultdict


def summarise(path):
    lines = open(path).read().splitlines()
    try:
        start = max(i for i, l in enumerate(lines) if l.startswith("---- run"))
    except ValueError:
        start = 0
    lines = lines[start:]
    lvl = defaultdict(float)
    cls = defaultdict(float)
    level = None
    for l in lines:
        m = re.match(r"\[lv\] level (\d+) (\S+)\s+([\d.]+) ms", l)
        if m:
            level = int(m.group(1))
            lvl[(level, m.group(2))] += float(m.group(3))
            continue
        m = re.match(r"\[lv\]\s+b(\d) (\S+)\s+nv=\d+\s+edges=\d+\s+([\d.]+) ms", l)
        if m and level is not None:
            cls[(level, "b" + m.group(1) + " " + m.group(2))] += float(m.group(3))
        m = re.match(r"\[lv\]\s+part (\S+)\s+([\d.]+) ms", l)
        if m and level is not None and m.group(1) != "setup":
            cls[(level, "  part " + m.group(1))] += float(m.group(2))
    return lvl, cls


def main():
    res = {p: summarise(p) for p in sys.argv[1:]}
    names = [p.split("/")[-1].replace(".err", "") for p in sys.argv[1:]]
    keys = sorted({k for lvl, _ in res.values() for k in lvl if k[1] in ("sweep", "modularity", "contract")})
    print(f"{'':24s}" + "".join(f"{n:>16s}" for n in names))
    for k in keys:
        print(f"L{k[0]} {k[1]:20s}" + "".join(f"{res[p][0].get(k, 0):16.2f}" for p in res))
    ckeys = sorted({k for _, cls in res.values() for k in cls})
    for k in ckeys:
        if k[0] > 2:
            continue
        print(f"L{k[0]} {k[1]:20s}" + "".join(f"{res[p][1].get(k, 0):16.2f}" for p in res))
    tot = {p: sum(v for k, v in res[p][0].items() if k[1] == "sweep") for p in res}
    print(f"{'sweep total':24s}" + "".join(f"{tot[p]:16.2f}" for p in res))


if __name__ == "__main__":
    main()
