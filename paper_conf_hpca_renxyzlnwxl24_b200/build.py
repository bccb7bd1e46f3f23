"""Build libdyo.so in-tree for sm_100a (nvcc; no JIT cache, so the .so travels with gpurun)."""
import os
import subprocess
import sys

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
OUT = os.path.join(HERE, "libdyo.so")
BUILD = os.path.join(HERE, "_build")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]
CU = ["pilot.cu", "pilot_tc.cu", "decode.cu", "plan.cu", "copy.cu", "partition.cu", "train.cu"]
CPP = ["api.cpp", "traverse.cpp", "nested.cpp"]


def _run(cmd):
    r = subprocess.run(cmd, capture_output=True, text=True)
    if r.returncode != 0:
        sys.stderr.write(r.stdout + r.stderr)
        raise RuntimeError("build failed: " + " ".join(cmd))
    return r.stdout + r.stderr


def build(force=False, verbose=False):
    os.makedirs(BUILD, exist_ok=True)
    srcs = [os.path.join(CSRC, f) for f in CU + CPP] + [os.path.join(CSRC, "dyo_internal.h"), os.path.join(CSRC, "decode_dev.cuh"), os.path.join(CSRC, "pilot_common.cuh"),
                                                       os.path.join(HERE, "..", "include", "dyo.h")]
    if not force and os.path.exists(OUT) and all(os.path.getmtime(OUT) >= os.path.getmtime(s) for s in srcs):
        build_cpu_baseline()
        return OUT
    objs = []
    for f in CU:
        o = os.path.join(BUILD, f + ".o")
        log = _run([NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC", "-Xptxas", "-v",
                    "-c", os.path.join(CSRC, f), "-o", o])
        if verbose:
            print(log)
        objs.append(o)
    for f in CPP:
        o = os.path.join(BUILD, f + ".o")
        _run([NVCC, "-O2", "-std=c++17", "-Xcompiler", "-fPIC,-Wall,-Wextra,-Werror=uninitialized,-Werror=init-self,-Wno-unused-parameter", "-x", "cu", *ARCH,
              "-c", os.path.join(CSRC, f), "-o", o])
        objs.append(o)
    _run([NVCC, *ARCH, "-shared", "-cudart", "static", "-o", OUT, *objs])
    build_cpu_baseline()
    return OUT


def build_cpu_baseline():
    """The compiled single-core CPU planner (baseline/cpu_planner.cpp): a bench/test baseline,
    not part of libdyo."""
    src = os.path.join(HERE, "..", "baseline", "cpu_planner.cpp")
    out = os.path.join(HERE, "..", "baseline", "libcpuplan.so")
    if os.path.exists(out) and os.path.getmtime(out) >= os.path.getmtime(src):
        return out
    _run(["g++", "-O3", "-march=x86-64-v3", "-std=c++17", "-shared", "-fPIC", "-o", out, src])
    return out


if __name__ == "__main__":
    print(build(force="--force" in sys.argv, verbose="-v" in sys.argv))
