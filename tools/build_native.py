"""Native build helpers (in-tree .so files; they travel to the GPU box with gpurun).

build_inputs()  -> inputs/libxkgen.so      (seeded generator, gcc -O2 -fopenmp)
build_oracle()  -> oracle/liboracle.so     (CPU oracle, gcc -O2 -fno-fast-math -ffp-contract=off)
build_xk()      -> paper_conf_sc_gautierl21_b200/libxk.so (product: nvcc sm_100a + C++ runtime)
"""
import glob
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _stale(target, sources):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(s) > t for s in sources)


def _run(cmd):
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True)
    if r.returncode != 0:
        raise RuntimeError("build failed: %s\n%s\n%s" % (" ".join(cmd), r.stdout, r.stderr))
    return r


def build_inputs(force=False):
    src = [os.path.join(ROOT, "inputs", "gen.c")]
    out = os.path.join(ROOT, "inputs", "libxkgen.so")
    if force or _stale(out, src):
        _run(["gcc", "-O2", "-fopenmp", "-fPIC", "-shared", "-o", out] + src + ["-lm"])
    return out


def build_oracle(force=False):
    src = [os.path.join(ROOT, "oracle", "oracle.c")]
    out = os.path.join(ROOT, "oracle", "liboracle.so")
    if force or _stale(out, src):
        _run(["gcc", "-std=c99", "-O2", "-fno-fast-math", "-ffp-contract=off", "-fopenmp",
              "-fPIC", "-shared", "-Wall", "-o", out] + src)
    return out


PKG = os.path.join(ROOT, "paper_conf_sc_gautierl21_b200")


def build_xk(force=False, verbose=False):
    csrc = os.path.join(PKG, "csrc")
    cu = sorted(glob.glob(os.path.join(csrc, "**", "*.cu"), recursive=True))
    cpp = sorted(glob.glob(os.path.join(csrc, "**", "*.cpp"), recursive=True))
    hdr = sorted(glob.glob(os.path.join(csrc, "**", "*.h"), recursive=True)) + \
        sorted(glob.glob(os.path.join(ROOT, "include", "*.h")))
    out = os.path.join(PKG, "libxk.so")
    if not (force or _stale(out, cu + cpp + hdr)):
        return out
    objdir = os.path.join(PKG, "build")
    os.makedirs(objdir, exist_ok=True)
    inc = ["-I", os.path.join(ROOT, "include"), "-I", csrc]
    objs = []
    procs = []
    for s in cu:
        o = os.path.join(objdir, os.path.basename(s) + ".o")
        objs.append(o)
        cmd = [NVCC] + ARCH + os.environ.get("XK_NVCC_FLAGS", "").split() + ["-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC",
                               "-Xptxas", "-v" if verbose else "-O3", "-c", s, "-o", o] + inc
        procs.append((cmd, subprocess.Popen(cmd, cwd=ROOT, stdout=subprocess.PIPE,
                                            stderr=subprocess.STDOUT, text=True)))
    for s in cpp:
        o = os.path.join(objdir, os.path.basename(s) + ".o")
        objs.append(o)
        cmd = ["g++", "-std=c++17", "-O2", "-fPIC", "-Wall", "-pthread", "-c", s, "-o", o,
               "-I", "/usr/local/cuda/include"] + inc
        procs.append((cmd, subprocess.Popen(cmd, cwd=ROOT, stdout=subprocess.PIPE,
                                            stderr=subprocess.STDOUT, text=True)))
    logs = []
    for cmd, p in procs:
        txt, _ = p.communicate()
        if p.returncode != 0:
            raise RuntimeError("build failed: %s\n%s" % (" ".join(cmd), txt))
        logs.append(txt)
    _run([NVCC] + ARCH + ["-shared", "-o", out] + objs +
         ["-Xcompiler", "-fPIC", "-cudart", "static", "-lpthread", "-ldl"])
    if verbose:
        print("\n".join(logs))
    return out


def build_example(force=False):
    """examples/xk_dgemm_example.c linked against libxk.so (the C ABI used from plain C)."""
    src = os.path.join(ROOT, "examples", "xk_dgemm_example.c")
    out = os.path.join(ROOT, "examples", "xk_dgemm_example")
    lib = build_xk()
    if force or _stale(out, [src, lib, os.path.join(ROOT, "include", "xk.h")]):
        _run(["gcc", "-O2", "-Wall", "-I", os.path.join(ROOT, "include"), src, "-L", PKG, "-lxk",
              "-Wl,-rpath," + PKG, "-lm", "-o", out])
    return out


def build_all(force=False):
    build_inputs(force)
    build_oracle(force)
    if os.path.isdir(os.path.join(PKG, "csrc")):
        build_xk(force)
        build_example(force)


if __name__ == "__main__":
    import sys
    build_all(force="--force" in sys.argv)
