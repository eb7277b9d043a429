"""Build the product library of another git revision for an A/B measurement on one box.

    python tools/ab_build.py REV NAME [-DMACRO=V ...]   ->  build/ab/NAME/liblouvain.so

REV = a git revision, or WT for the working tree's sources; -D: compile-time variants.

Run the other arm with LOUVAIN_LIB=build/ab/NAME/liblouvain.so (paper_conf_ipps_naimmht17_b200
loads that file instead of the in-tree build).  The C-ABI header is taken from the working tree.
"""
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, os.path.join(ROOT, "tools"))
import build  # noqa: E402


def main():
    rev, name = sys.argv[1], sys.argv[2]
    defines = [a[2:] for a in sys.argv[3:] if a.startswith("-D")]
    src = os.path.join(ROOT, "build", "ab", name, "csrc")
    os.makedirs(src, exist_ok=True)
    rel = "paper_conf_ipps_naimmht17_b200/csrc"
    files = [] if rev == "WT" else subprocess.run(["git", "ls-tree", "--name-only", f"{rev}:{rel}"], cwd=ROOT,
                                                  check=True, capture_output=True, text=True).stdout.split()
    if rev == "WT":
        files = sorted(os.listdir(os.path.join(ROOT, rel)))
    for f in files:
        if rev == "WT":
            with open(os.path.join(ROOT, rel, f), "rb") as fh:
                data = fh.read()
        else:
            data = subprocess.run(["git", "show", f"{rev}:{rel}/{f}"], cwd=ROOT, check=True,
                                  capture_output=True).stdout
        with open(os.path.join(src, f), "wb") as fh:
            fh.write(data)
    out = os.path.join(ROOT, "build", "ab", name, "liblouvain.so")
    build.build_louvain(force=True, d=src, out=out, objdir=os.path.join(ROOT, "build", "ab", name, "obj"),
                        defines=defines)
    # only the library travels to the GPU box (gpurun snapshots are capped at 512 MiB)
    shutil.rmtree(os.path.join(ROOT, "build", "ab", name, "obj"), ignore_errors=True)
    shutil.rmtree(src, ignore_errors=True)
    print(out)


if __name__ == "__main__":
    main()
