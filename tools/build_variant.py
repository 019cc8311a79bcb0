"""Build an A/B or instrumented copy of liblime.so with extra nvcc flags into its own directory
(e.g. -DLIME_TRACE); point LIME_LIBRARY at the result. Not part of the product build.

    python tools/build_variant.py OUT_DIR -DLIME_TRACE [...]
"""
import os
import subprocess
import sys
from concurrent.futures import ThreadPoolExecutor

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_pldi_dubachcrbf12_b200 import build as b  # noqa: E402


def main():
    out, extra = sys.argv[1], sys.argv[2:]
    os.makedirs(out, exist_ok=True)

    def cc(src):
        obj = os.path.join(out, os.path.basename(src).replace(".cu", ".o"))
        r = subprocess.run([b.nvcc(), *b.ARCH, *b.NVCC_FLAGS, *extra, "-c", src, "-o", obj], capture_output=True, text=True)
        if r.returncode:
            raise RuntimeError(r.stderr)
        return obj

    with ThreadPoolExecutor(8) as ex:
        objs = list(ex.map(cc, b._sources()))
    lib = os.path.join(out, "liblime.so")
    subprocess.run([b.nvcc(), *b.ARCH, "-shared", "-cudart", "static", "-o", lib, *objs], check=True)
    print(lib)


if __name__ == "__main__":
    main()
