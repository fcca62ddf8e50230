"""Build an A/B variant of libbullet.so with extra nvcc defines (experiments
only): python scripts/build_variant.py OUT.so -DDEC_NCW=6 -DDEC_DEPTH=4
Load it with BULLET_LIB=OUT.so."""
import concurrent.futures as cf
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
from paper_conf_asplos_0001xc0l026_b200 import build as B  # noqa: E402


def main():
    out, extra = os.path.abspath(sys.argv[1]), sys.argv[2:]
    odir = out + ".objs"
    os.makedirs(odir, exist_ok=True)

    def comp(src):
        obj = os.path.join(odir, os.path.basename(src) + ".o")
        r = subprocess.run([B.NVCC, *B.ARCH, *B.FLAGS, *extra, "-c", src, "-o", obj], capture_output=True, text=True)
        if r.returncode:
            raise RuntimeError(r.stderr)
        return obj
    with cf.ThreadPoolExecutor(8) as ex:
        objs = list(ex.map(comp, B.sources()))
    r = subprocess.run([B.NVCC, *B.ARCH, "-shared", "-o", out, *objs, "-ldl"], capture_output=True, text=True)
    if r.returncode:
        raise RuntimeError(r.stderr)
    print(out)


if __name__ == "__main__":
    main()
