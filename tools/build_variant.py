"""Build an A/B variant of libspmv.so: the csrc tree copied to build/variants/NAME with
literal source substitutions applied, compiled with the product flags into
build/variants/NAME/libspmv.so.  Load it with SPMV_LIB_PATH=<that path> (spmv.lib()).

usage: python tools/build_variant.py NAME FILE 'OLD' 'NEW' [FILE 'OLD' 'NEW' ...]
"""
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

from paper_conf_ipps_nisassvs18_b200 import build_lib  # noqa: E402


def main():
    name, subs = sys.argv[1], sys.argv[2:]
    if len(subs) % 3:
        raise SystemExit(__doc__)
    out = os.path.join(ROOT, "build", "variants", name)
    src = os.path.join(out, "csrc")
    shutil.rmtree(out, ignore_errors=True)
    shutil.copytree(build_lib.CSRC, src)
    inc = os.path.join(ROOT, "build", "variants", "include")      # csrc includes ../../include/spmv.h
    shutil.rmtree(inc, ignore_errors=True)
    shutil.copytree(os.path.join(ROOT, "include"), inc)
    for i in range(0, len(subs), 3):
        f, old, new = subs[i:i + 3]
        p = os.path.join(src, f)
        txt = open(p).read()
        if old not in txt:
            raise SystemExit(f"{f}: substitution source not found: {old!r}")
        open(p, "w").write(txt.replace(old, new))
    objs = []
    procs = []
    for s in sorted(os.listdir(src)):
        if s.endswith(".cu"):
            o = os.path.join(out, s + ".o")
            objs.append(o)
            procs.append(subprocess.Popen(["nvcc", *build_lib.NVCC_FLAGS, "-I", os.path.join(ROOT, "include"),
                                           "-c", os.path.join(src, s), "-o", o],
                                          stdout=subprocess.DEVNULL, stderr=subprocess.PIPE))
    for p in procs:
        _, err = p.communicate()
        if p.returncode:
            raise SystemExit(err.decode())
    lib = os.path.join(out, "libspmv.so")
    subprocess.check_call(["nvcc", "-gencode", "arch=compute_100a,code=sm_100a", "-shared", "-Xcompiler", "-fPIC",
                           "-o", lib, *objs, "-lcudart_static", "-lrt", "-ldl", "-lpthread"])
    print(lib)


if __name__ == "__main__":
    main()
