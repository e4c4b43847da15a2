"""Build libefit_b200.so (sm_100a) in-tree with nvcc.  Called by __graft_entry__.build()."""
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
ROOT = os.path.dirname(HERE)
CSRC = os.path.join(HERE, "csrc")
LIB = os.path.join(HERE, "libefit_b200.so")
SOURCES = ["efit_api.cu", "efit_kernels.cu", "efit_steps.cu"]
# per-source flags: the steps_ kernels take discrete decisions from fp64 expressions that must round
# exactly as written (no FMA contraction anywhere in that translation unit)
SOURCE_FLAGS = {"efit_steps.cu": ["-fmad=false"]}
HEADERS = ["efit_internal.h", "efit_device.cuh"]

NVCC_FLAGS = ["-O3", "-std=c++17", "-gencode", "arch=compute_100a,code=sm_100a", "-lineinfo",
              "-Xptxas", "-v", "-Xcompiler", "-fPIC", "--expt-relaxed-constexpr",
              "-I" + os.path.join(ROOT, "include"), "-I" + CSRC]


def _stale() -> bool:
    if not os.path.exists(LIB):
        return True
    t = os.path.getmtime(LIB)
    deps = [os.path.join(CSRC, f) for f in SOURCES + HEADERS] + [os.path.join(ROOT, "include", "efit.h")]
    return any(os.path.getmtime(d) > t for d in deps)


def build(force: bool = False, verbose: bool = False, defines=(), out: str = LIB) -> str:
    """Compile both sources and link `out`.  `defines` (e.g. ["EFIT_SYM_UNR=3"]) build a tuning
    variant into another file (the default library is always the untuned default build)."""
    if not force and not defines and out == LIB and not _stale():
        return LIB
    objs = []
    log = []
    for src in SOURCES:
        tag = "" if out == LIB else "." + os.path.basename(out).replace(".so", "")
        obj = os.path.join(CSRC, src.replace(".cu", tag + ".o"))
        hdrs = [os.path.join(CSRC, h) for h in HEADERS] + [os.path.join(ROOT, "include", "efit.h"), __file__]
        if (not force and not defines and os.path.exists(obj) and
                all(os.path.getmtime(obj) > os.path.getmtime(d) for d in hdrs + [os.path.join(CSRC, src)])):
            objs.append(obj)  # object up to date (incremental build)
            continue
        cmd = ["nvcc", *NVCC_FLAGS, *SOURCE_FLAGS.get(src, []), *["-D" + d for d in defines], "-c",
               os.path.join(CSRC, src), "-o", obj]
        r = subprocess.run(cmd, capture_output=True, text=True)
        log.append(r.stdout + r.stderr)
        if r.returncode != 0:
            sys.stderr.write(r.stdout + r.stderr)
            raise RuntimeError(f"nvcc failed on {src}")
        objs.append(obj)
    tmp = out + f".tmp{os.getpid()}"
    cmd = ["nvcc", "-shared", "-gencode", "arch=compute_100a,code=sm_100a", "-o", tmp, *objs, "-lcudart"]
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("nvcc link failed")
    os.replace(tmp, out)
    if out == LIB:
        with open(os.path.join(CSRC, "ptxas.log"), "w") as f:
            f.write("\n".join(log))
    if verbose:
        print("\n".join(log))
    return out


if __name__ == "__main__":
    build(force="--force" in sys.argv, verbose=True)
