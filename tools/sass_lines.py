"""Per-source-line totals of an ncu source page (SASS rows) for one kernel:
instructions executed, thread instructions (-> active lanes), stall samples.
The SASS offsets are mapped to lines with `nvdisasm -g` of the same build.

    python tools/sass_lines.py gpurun_out/x.sass.csv build/louvain/lv_sweep.cu.o <mangled-substring> [top]
"""
import csv
import os
import re
import subprocess
import sys
import tempfile
from collections import defaultdict


def line_map(obj, key):
    d = tempfile.mkdtemp()
    subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(obj)], cwd=d, capture_output=True)
    cub = [f for f in os.listdir(d) if f.endswith(".cubin")][0]
    out = subprocess.run(["nvdisasm", "-g", "-c", os.path.join(d, cub)], capture_output=True, text=True).stdout
    m, cur, inside, line = {}, None, False, None
    for s in out.splitlines():
        if s.startswith("//--------------------- .text."):
            inside = key in s
            continue
        if not inside:
            continue
        g = re.search(r'//## File ".*?/([^/"]+)", line (\d+)', s)
        if g:
            line = f"{g.group(1)}:{g.group(2)}"
            continue
        g = re.match(r"\s*/\*([0-9a-f]{4,})\*/", s)
        if g:
            m[int(g.group(1), 16)] = line
    return m


def main():
    path, obj, key = sys.argv[1], sys.argv[2], sys.argv[3]
    top = int(sys.argv[4]) if len(sys.argv) > 4 else 25
    rows = list(csv.reader(open(path)))
    hdr = rows[1]
    ix = {h: i for i, h in enumerate(hdr)}
    base = None
    lm = line_map(obj, key)
    agg = defaultdict(lambda: [0, 0, 0])
    tot = [0, 0, 0]
    for r in rows[2:]:
        if len(r) < len(hdr):
            continue
        try:
            a = int(r[ix["Address"]], 16)
        except ValueError:  # the next kernel's section (several launches in one file): first only
            break
        base = a if base is None else base
        off = a - base
        ln = lm.get(off, "?")
        ie, te, st = int(r[ix["Instructions Executed"]] or 0), int(r[ix["Thread Instructions Executed"]] or 0), \
            int(r[ix["Warp Stall Sampling (All Samples)"]] or 0)
        for k, v in enumerate((ie, te, st)):
            agg[ln][k] += v
            tot[k] += v
    print(f"total warp instr {tot[0]:.3e}  thread instr {tot[1]:.3e}  lanes/instr {tot[1] / max(tot[0], 1):.1f}  "
          f"stall samples {tot[2]}")
    for ln, (ie, te, st) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
        print(f"{ln:>18}  instr {100 * ie / tot[0]:5.1f}%  lanes {te / max(ie, 1):5.1f}  stall {100 * st / max(tot[2], 1):5.1f}%")


if __name__ == "__main__":
    main()
