"""Build an A/B variant of libb2cl.so with extra -D defines on one kernel source:
    python tools/build_variant.py NAME [--src kernels/rect.cu] [--file path.cu] -DB2CL_C3_XPT=8 ...
writes build/variants/NAME.so (use with B2CL_LIB=...).  --src picks the source
the defines apply to (default kernels/sample.cu); --file compiles another file
in its place (e.g. an older revision saved next to it)."""
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from paper_conf_sc_kimdjjl15_b200 import build as B  # noqa: E402


def main():
    args = sys.argv[1:]
    name = args.pop(0)
    target, repl = "kernels/sample.cu", None
    while args and args[0] in ("--src", "--file"):
        flag, val = args.pop(0), args.pop(0)
        if flag == "--src":
            target = val
        else:
            repl = val
    defs = args
    B.build()
    out_dir = os.path.join(B.ROOT, "build", "variants")
    os.makedirs(out_dir, exist_ok=True)
    objs = []
    for src in B.SOURCES:
        obj = os.path.join(B.BUILD, src.replace("/", "_") + ".o")
        if src == target:
            obj = os.path.join(out_dir, f"{name}_{os.path.basename(src)}.o")
            path = repl or os.path.join(B.CSRC, src)
            subprocess.run([B.NVCC, *B.ARCH, *B.FLAGS, *defs, "-x", "cu", "-c", path, "-o", obj],
                           check=True)
        objs.append(obj)
    lib = os.path.join(out_dir, f"{name}.so")
    subprocess.run([B.NVCC, *B.ARCH, "-shared", "-cudart", "static", "-o", lib, *objs, "-lpthread",
                    "-ldl", "-lrt"], check=True)
    print(lib)


if __name__ == "__main__":
    main()
