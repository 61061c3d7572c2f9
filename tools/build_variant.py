"""Build a variant of libslate.so with extra -D flags into build/variants/ (experiments only).

    python tools/build_variant.py NAME -DFOO=1 [-DBAR=2 ...]   ->  build/variants/libslate_NAME.so
Run a tool against it with SLATE_LIB=build/variants/libslate_NAME.so."""
import concurrent.futures as cf
import glob
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
C = os.path.join(ROOT, "paper_conf_ipps_allenf019_b200", "csrc")
OUT = os.path.join(ROOT, "build", "variants")
NVCC = "/usr/local/cuda/bin/nvcc"
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def main():
    name, defs = sys.argv[1], sys.argv[2:]
    os.makedirs(OUT, exist_ok=True)
    srcs = [s for s in sorted(glob.glob(C + "/*.cu") + glob.glob(C + "/*.cpp")) if not os.path.basename(s).startswith("slated")]

    def comp(src):
        o = os.path.join(OUT, "%s_%s.o" % (name, os.path.basename(src)))
        cmd = [NVCC] + ARCH + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-I", os.path.join(ROOT, "include"),
                               "--expt-relaxed-constexpr"] + defs + ["-c", src, "-o", o]
        r = subprocess.run(cmd, capture_output=True, text=True)
        if r.returncode:
            raise RuntimeError(r.stderr)
        return o

    with cf.ThreadPoolExecutor(8) as ex:
        objs = list(ex.map(comp, srcs))
    lib = os.path.join(OUT, "libslate_%s.so" % name)
    r = subprocess.run([NVCC] + ARCH + ["-shared", "-o", lib] + objs + ["-lpthread", "-ldl", "-lrt"], capture_output=True, text=True)
    if r.returncode:
        raise RuntimeError(r.stderr)
    print(lib)


if __name__ == "__main__":
    main()
