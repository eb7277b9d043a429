"""Per-kernel-family time shares of an ncu launch list (gpu__time_duration.sum) of the
bench command: which kernels a C5 run spends its device time in.  Cold-cache,
serialised times: shares, not absolutes.

    python tools/launch_shares.py profiles/r01_bench_c5_launches_v6.csv
"""
import collections
import csv
import re
import sys


def family(name: str) -> str:
    m = re.match(r"(?:void )?(?:lv::<unnamed>::|cub::|lv::)?([A-Za-z_0-9]+)", name)
    base = m.group(1) if m else name
    if name.startswith("cub::") or "cub::" in name[:20]:
        return "cub::" + base
    return base


def main():
    rows, hdr = [], None
    for r in csv.reader(open(sys.argv[1])):
        if r and r[0] == "ID":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            d = dict(zip(hdr, r))
            if d["Metric Name"] == "gpu__time_duration.sum":
                rows.append(d)
    unit = rows[0]["Metric Unit"] if rows else "ns"
    scale = {"ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "nsecond": 1e-6, "ms": 1.0, "msecond": 1.0}.get(unit, 1e-6)
    tot = collections.Counter()
    cnt = collections.Counter()
    for d in rows:
        f = family(d["Kernel Name"])
        tot[f] += float(d["Metric Value"].replace(",", "")) * scale
        cnt[f] += 1
    all_ms = sum(tot.values())
    print(f"{len(rows)} launches, {all_ms:.1f} ms (ncu, serialised; the bench command = warm-up + timed + e2e runs)")
    for f, ms in tot.most_common(40):
        print(f"  {100 * ms / all_ms:5.1f}%  {ms:9.1f} ms  {cnt[f]:5d} x  {f}")


if __name__ == "__main__":
    main()
