"""Build every native artefact in-tree (called by __graft_entry__.build()).

* gen/libsievegen.so      -- synthetic trace generator (host; gcc + OpenMP)
* oracle/libsieve_oracle.so -- the CPU oracle (test infrastructure; gcc, -ffp-contract=off)
* paper_conf_ispass_naderantahanse23_b200/libsieve.so -- the product: sm_100a kernels + C-ABI
"""
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PKG = os.path.join(ROOT, "paper_conf_ispass_naderantahanse23_b200")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")
ARCH = ["-gencode", "arch=compute_100a,code=sm_100a"]


def _run(cmd):
    print("+", " ".join(cmd), flush=True)
    subprocess.check_call(cmd, cwd=ROOT)


def _stale(target, sources):
    if not os.path.exists(target):
        return True
    t = os.path.getmtime(target)
    return any(os.path.getmtime(s) > t for s in sources)


def build_gen(force=False):
    src = [os.path.join(ROOT, "gen", "gen_host.c"), os.path.join(ROOT, "gen", "sieve_gen.h")]
    out = os.path.join(ROOT, "gen", "libsievegen.so")
    if force or _stale(out, src):
        _run(["gcc", "-O2", "-std=c11", "-fopenmp", "-fPIC", "-shared", "-o", out, src[0], "-lm"])
    return out


def build_oracle(force=False):
    src = [os.path.join(ROOT, "oracle", "sieve_oracle.c")]
    out = os.path.join(ROOT, "oracle", "libsieve_oracle.so")
    if force or _stale(out, src):
        # no -ffast-math, no FP contraction: every fp64 step is the IEEE operation written
        _run(["gcc", "-O2", "-std=c11", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared",
              "-o", out, src[0], "-lm"])
    return out


def cuda_sources():
    d = os.path.join(PKG, "csrc")
    return sorted(os.path.join(d, f) for f in os.listdir(d) if f.endswith((".cu", ".cpp")))


def build_lib(force=False):
    srcs = cuda_sources()
    hdrs = [os.path.join(PKG, "csrc", f) for f in os.listdir(os.path.join(PKG, "csrc"))
            if f.endswith((".cuh", ".h"))] + [os.path.join(ROOT, "include", "sieve.h")]
    out = os.path.join(PKG, "libsieve.so")
    if not (force or _stale(out, srcs + hdrs)):
        return out
    objdir = os.path.join(ROOT, "build", "obj")
    os.makedirs(objdir, exist_ok=True)
    objs = []
    for s in srcs:
        o = os.path.join(objdir, os.path.basename(s) + ".o")
        objs.append(o)
        if not force and not _stale(o, [s] + hdrs):
            continue
        _run([NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-ffp-contract=off",
              "-I", os.path.join(ROOT, "include"), "-I", os.path.join(PKG, "csrc"),
              "-x", "cu" if s.endswith(".cu") else "c++", "-c", s, "-o", o])
    _run([NVCC, *ARCH, "-shared", "-o", out, *objs, "-lcudart_static", "-ldl", "-lpthread", "-lrt"])
    return out


def build_variant(name, source, defines):
    """A/B builds: the library with some sources (a file name or a list) compiled under extra
    -D flags, written to build/variants/libsieve_<name>.so (select it with SIEVE_LIB_PATH)."""
    sources = [source] if isinstance(source, str) else list(source)
    build_lib()
    objdir = os.path.join(ROOT, "build", "obj")
    vdir = os.path.join(ROOT, "build", "variants")
    os.makedirs(vdir, exist_ok=True)
    objs = []
    for s in cuda_sources():
        o = os.path.join(objdir, os.path.basename(s) + ".o")
        if os.path.basename(s) in sources:
            o = os.path.join(vdir, f"{name}_{os.path.basename(s)}.o")
            _run([NVCC, *ARCH, "-O3", "-lineinfo", "-std=c++17", "-Xcompiler", "-fPIC,-ffp-contract=off",
                  *[f"-D{d}" for d in defines], "-I", os.path.join(ROOT, "include"),
                  "-I", os.path.join(PKG, "csrc"), "-x", "cu", "-c", s, "-o", o])
        objs.append(o)
    out = os.path.join(vdir, f"libsieve_{name}.so")
    _run([NVCC, *ARCH, "-shared", "-o", out, *objs, "-lcudart_static", "-ldl", "-lpthread", "-lrt"])
    return out


def build_all(force=False):
    build_gen(force)
    build_oracle(force)
    build_lib(force)


if __name__ == "__main__":
    build_all(force="--force" in sys.argv)
