"""Build an A/B variant of libb2cl.so with extra -D defines on sample.cu:
    python tools/build_variant.py NAME -DB2CL_C3_XPT=8 ...
writes build/variants/NAME.so (use with B2CL_LIB=...)."""
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

from paper_conf_sc_kimdjjl15_b200 import build as B  # noqa: E402


def main():
    name, defs = sys.argv[1], sys.argv[2:]
    B.build()
    out_dir = os.path.join(B.ROOT, "build", "variants")
    os.makedirs(out_dir, exist_ok=True)
    objs = []
    for src in B.SOURCES:
        obj = os.path.join(B.BUILD, src.replace("/", "_") + ".o")
        if src == "kernels/sample.cu":
            obj = os.path.join(out_dir, f"{name}_sample.o")
            subprocess.run([B.NVCC, *B.ARCH, *B.FLAGS, *defs, "-x", "cu", "-c",
                            os.path.join(B.CSRC, src), "-o", obj], check=True)
        objs.append(obj)
    lib = os.path.join(out_dir, f"{name}.so")
    subprocess.run([B.NVCC, *B.ARCH, "-shared", "-cudart", "static", "-o", lib, *objs, "-lpthread",
                    "-ldl", "-lrt"], check=True)
    print(lib)


if __name__ == "__main__":
    main()
