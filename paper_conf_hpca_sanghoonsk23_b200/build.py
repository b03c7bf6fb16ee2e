"""Build libccube.so in-tree with nvcc for sm_100a (no GPU needed).

    python -m paper_conf_hpca_sanghoonsk23_b200.build

Flags: -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo; no --use_fast_math,
no -ftz (the fp32/bf16 results must be bit-exact to the oracle).
cudart is linked statically and the driver API is reached through
cudaGetDriverEntryPoint, so the library loads on a machine without a GPU (the
CPU tests check its exports) and fails loudly only when it is asked to compute.
"""

import os
import shutil
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libccube.so")
INCLUDE = os.path.join(ROOT, "include")

ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
NVCC_FLAGS = ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-fvisibility=hidden",
              "-Xptxas", "-v", "--expt-relaxed-constexpr"]
SOURCES = ["tree_allreduce.cu", "runtime.cc", "trees.cc", "plan.cc"]


def nvcc() -> str:
    for cand in (os.environ.get("NVCC"), shutil.which("nvcc"), "/usr/local/cuda/bin/nvcc"):
        if cand and os.path.exists(cand):
            return cand
    raise RuntimeError("nvcc not found")


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in os.listdir(CSRC)] + [os.path.join(INCLUDE, "ccube.h")]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, target: str = LIB, defines=()) -> str:
    """Compile and link the library.  ``target`` / ``defines`` (-D macros) build
    experiment variants (tools/experiments); the product is the default in-tree LIB."""
    if target == LIB and not defines and not force and not _stale():
        return LIB
    objs = []
    tmp = os.path.join(HERE, "build", os.path.basename(target).replace(".so", ""))
    os.makedirs(tmp, exist_ok=True)
    for src in SOURCES:
        obj = os.path.join(tmp, os.path.splitext(src)[0] + ".o")
        lang = [] if src.endswith(".cu") else ["-x", "cu"]
        cmd = [nvcc(), *ARCH, *NVCC_FLAGS, *[f"-D{d}" for d in defines], "-I", INCLUDE,
               "-I", CSRC, *lang, "-c",
               os.path.join(CSRC, src), "-o", obj]
        out = subprocess.run(cmd, capture_output=True, text=True)
        if out.returncode != 0:
            raise RuntimeError(f"nvcc failed for {src}:\n{out.stdout}\n{out.stderr}")
        if verbose:
            sys.stderr.write(out.stderr)
        objs.append(obj)
    cmd = [nvcc(), *ARCH, "-shared", "-cudart", "static", "-o", target + ".tmp", *objs,
           "-Xlinker", "--version-script=" + os.path.join(CSRC, "ccube.map"),
           "-lpthread", "-ldl", "-lrt"]
    out = subprocess.run(cmd, capture_output=True, text=True)
    if out.returncode != 0:
        raise RuntimeError(f"link failed:\n{out.stdout}\n{out.stderr}")
    os.replace(target + ".tmp", target)
    return target


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose=True))
