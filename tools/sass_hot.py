"""Summarise an `ncu --page source --csv --print-source sass` export: opcode mix
and the instructions with the most stall samples (first kernel section only).

    python tools/sass_hot.py file.csv [section]
"""
import collections
import csv
import sys


def sections(path):
    cur = None
    hdr = None
    for r in csv.reader(open(path)):
        if r and r[0] == "Kernel Name":
            if cur:
                yield cur
            cur = {"name": r[1], "rows": []}
            continue
        if r and r[0] == "Address":
            hdr = r
            continue
        if cur is not None and hdr and len(r) == len(hdr):
            cur["rows"].append(dict(zip(hdr, r)))
    if cur:
        yield cur


def main():
    secs = list(sections(sys.argv[1]))
    k = int(sys.argv[2]) if len(sys.argv) > 2 else 0
    s = secs[k]
    data = s["rows"]
    f = lambda d, key: float(d.get(key) or 0)  # noqa: E731
    tot = sum(f(d, "Instructions Executed") for d in data) or 1
    tst = sum(f(d, "Warp Stall Sampling (All Samples)") for d in data) or 1
    print(s["name"][:120], f"warp-instr={tot:.3g}", f"samples={tst:.0f}")
    op, ops = collections.Counter(), collections.Counter()
    for d in data:
        toks = d["Source"].split()
        o = toks[1] if toks and toks[0].startswith("@") and len(toks) > 1 else (toks[0] if toks else "?")
        o = o.split(".")[0]
        op[o] += f(d, "Instructions Executed")
        ops[o] += f(d, "Warp Stall Sampling (All Samples)")
    for o, c in op.most_common(22):
        print(f"  {o:10s} instr {c / tot * 100:5.1f}%  stall {ops[o] / tst * 100:5.1f}%")
    print("  --- top stall sites")
    for i, d in sorted(enumerate(data), key=lambda x: -f(x[1], "Warp Stall Sampling (All Samples)"))[:25]:
        reasons = sorted(((f(d, kk), kk) for kk in d if kk.startswith("stall_") and "Not Issued" not in kk),
                         reverse=True)[:2]
        rs = " ".join(f"{kk[6:]}={v:.0f}" for v, kk in reasons if v)
        print(f"  {i:5d} {d['Source'].strip()[:58]:58s} ex {f(d, 'Instructions Executed') / tot * 100:5.2f}% "
              f"st {f(d, 'Warp Stall Sampling (All Samples)') / tst * 100:5.1f}% {rs}")


if __name__ == "__main__":
    main()
