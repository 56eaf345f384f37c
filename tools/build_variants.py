"""A/B builds of libcswap.so with compile-time switches, for measuring kernel design choices on
the box in one call:  python tools/build_variants.py TAG=-DFLAG=V[,-DFLAG2=V] ...
Each lands in paper_conf_cluster_chenhzchysc21_b200/variants/libcswap_TAG.so; select it with
CSWAP_LIB_VARIANT=TAG (cswap.py)."""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_cluster_chenhzchysc21_b200 import build as B  # noqa: E402


def main():
    out_dir = os.path.join(B.PKG, "variants")
    os.makedirs(out_dir, exist_ok=True)
    for spec in sys.argv[1:]:
        tag, flags = spec.split("=", 1)
        defs = [f for f in flags.split(",") if f]
        obj_dir = os.path.join(B.OBJ, "var_" + tag)
        os.makedirs(obj_dir, exist_ok=True)
        objs = []
        for src in B.sources():
            obj = os.path.join(obj_dir, os.path.basename(src) + ".o")
            subprocess.run([B.NVCC, *B.ARCH, *B.FLAGS, *defs, "-c", src, "-o", obj], check=True)
            objs.append(obj)
        lib = os.path.join(out_dir, f"libcswap_{tag}.so")
        subprocess.run([B.NVCC, *B.ARCH, "-shared", "-cudart", "static", "-o", lib, *objs, "-lpthread"], check=True)
        print(lib)


if __name__ == "__main__":
    main()
