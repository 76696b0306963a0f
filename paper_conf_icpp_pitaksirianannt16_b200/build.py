"""Build libtbs.so (the C-ABI library) in-tree with nvcc for sm_100a."""
import glob
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
LIB = os.path.join(HERE, "libtbs.so")
SRCS = [os.path.join(HERE, "csrc", f) for f in ("tbs_api.cu",)]
DEPS = SRCS + sorted(glob.glob(os.path.join(HERE, "csrc", "*.cuh"))) + [os.path.join(ROOT, "include", "tbs.h")]
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
FLAGS = ["-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo", "-std=c++17",
         "-Xcompiler", "-fPIC", "-shared", "-cudart", "static", "-Xptxas", "-v"]


def build(force=False, verbose=False, out=None, defines=()):
    """Build libtbs.so (or, for A/B experiments, a variant at `out` with -D`defines`)."""
    target = out or LIB
    if not force and os.path.exists(target) and all(os.path.getmtime(target) >= os.path.getmtime(d) for d in DEPS):
        return target
    tmp = target + f".tmp{os.getpid()}"
    extra = [d[len("NVCC:"):] for d in defines if d.startswith("NVCC:")]   # A/B builds: raw nvcc flags
    defs = [f"-D{d}" for d in defines if not d.startswith("NVCC:")]
    cmd = [NVCC] + FLAGS + extra + defs + ["-I", os.path.join(ROOT, "include"), "-o", tmp] + SRCS
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc failed building libtbs.so")
    if out is None:
        with open(os.path.join(HERE, "csrc", "ptxas_report.txt"), "w") as f:
            f.write(r.stderr)
    if verbose:
        sys.stderr.write(r.stderr)
    os.replace(tmp, target)
    return target


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
